// common.cuh -- host-side helpers shared by the libcudanp translation units:
// status/error text, argument checks, launch-shape computation.
#pragma once
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <cuda_runtime.h>

#include "../../include/cudanp.h"

namespace cudanp {

// Thread-local detail for cudanp_last_error().
void set_error(const char* fmt, ...);

inline int fail_invalid(const char* what) {
  set_error("invalid argument: %s", what);
  return CUDANP_ERR_INVALID;
}

inline int check_launch(const char* what) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    set_error("%s: %s", what, cudaGetErrorString(e));
    return CUDANP_ERR_CUDA;
  }
  return CUDANP_OK;
}

inline bool valid_S(int S) {
  return S == 1 || S == 2 || S == 4 || S == 8 || S == 16 || S == 32;
}
// Inter-warp teams need not be a power of two (the padding limit of
// intra-warp NP "can be removed" for inter-warp NP; Fig 12, uses 3, 5,
// 10 and 15): these S are built for the inter-warp map of TMV, MV, the
// batched reduce and the batched scan (and the LE kernel, np_le.cu).
inline bool valid_inter_S(int S) { return S == 3 || S == 5 || S == 10 || S == 15; }
template <int S> constexpr bool kPow2 = S > 0 && (S & (S - 1)) == 0;

// Teams larger than a warp (S/32 consecutive warps; shfl within each warp,
// shared memory across them): batched reduce/scan and MV with the intra-warp
// (consecutive-thread) map, TMV with the inter-warp map for S <= 128.
inline bool valid_big_S(int S) { return S == 64 || S == 128 || S == 256 || S == 512 || S == 1024; }

// Teams larger than a CTA (batched reduce and scan, MV): one thread-block cluster of 8
// CTAs of S/8 threads (np_cluster.cu).
inline bool valid_cluster_S(int S) { return S == 2048 || S == 4096 || S == 8192; }

inline bool aligned16(const void* p) { return ((uintptr_t)p & 15u) == 0; }

// SM count of the current device (cached per device ordinal).
int sm_count();

// Programmatic dependent launch on/off for the hot-path kernels (default on;
// CUDANP_PDL=0 in the environment turns it off, for A/B measurements).
bool pdl_enabled();

// Launch `kern` with programmatic stream serialization allowed (when enabled):
// the kernel must begin with pdl_entry() (np_team.cuh).
// `allow` = false launches without the attribute (the kernel's
// griddepcontrol instructions are then no-ops and it starts after its
// predecessor completes, as an ordinary stream launch).
template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl_if(bool allow, void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem,
                                 cudaStream_t st, Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = (allow && pdl_enabled()) ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
}
template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem,
                              cudaStream_t st, Args... args) {
  return launch_pdl_if(true, kern, grid, block, smem, st, args...);
}


// Grid for a persistent grid-stride kernel: enough CTAs to cover `work_ctas`
// units of CTA work, capped at (resident CTAs per SM) x (SM count), so the
// grid is a whole number of waves.
template <class K>
inline int64_t persistent_grid(K kernel, int block_threads, size_t dyn_smem, int64_t work_ctas) {
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, block_threads, dyn_smem) !=
          cudaSuccess ||
      per_sm < 1) {
    cudaGetLastError();
    per_sm = 1;
  }
  int64_t cap = (int64_t)per_sm * sm_count();
  if (work_ctas < 1) work_ctas = 1;
  return work_ctas < cap ? work_ctas : cap;
}

// Persistent intra-warp launches take K consecutive warp tiles per warp step
// (K tiles of loads in flight).  When there are too few tiles to give every
// resident warp K of them, the K = 1 instantiation is launched instead so a
// few-item launch still spreads over every SM (a compile-time K keeps the
// register count, and so the occupancy, of the common case).
template <class Kn>
inline bool few_tiles(Kn kernel_k, int block_threads, int64_t ntiles, int K) {
  const int64_t cap_ctas = persistent_grid(kernel_k, block_threads, 0, INT64_MAX / 4);
  return 2 * ntiles < cap_ctas * (block_threads / 32) * K;
}

template <class K>
inline void kernel_attrs(K kernel, int* regs, int* smem) {
  cudaFuncAttributes a;
  if (cudaFuncGetAttributes(&a, kernel) == cudaSuccess) {
    if (regs) *regs = a.numRegs;
    if (smem) *smem = (int)a.sharedSizeBytes;
  } else {
    cudaGetLastError();
  }
}

// Launch-shape record filled by the dispatchers when info-only is requested.
struct LaunchInfo {
  int block_threads = 0;
  int64_t grid = 0;
  int regs = 0;
  int smem = 0;
  int map = 0;
};

}  // namespace cudanp

// Dispatch a runtime team size to a compile-time constant `kS`.
#define CUDANP_DISPATCH_S(S, ...)                        \
  switch (S) {                                           \
    case 1: { constexpr int kS = 1; __VA_ARGS__; } break;   \
    case 2: { constexpr int kS = 2; __VA_ARGS__; } break;   \
    case 4: { constexpr int kS = 4; __VA_ARGS__; } break;   \
    case 8: { constexpr int kS = 8; __VA_ARGS__; } break;   \
    case 16: { constexpr int kS = 16; __VA_ARGS__; } break; \
    case 32: { constexpr int kS = 32; __VA_ARGS__; } break; \
    default: return fail_invalid("S must be one of 1,2,4,8,16,32"); \
  }
// The non-power-of-two inter-warp team sizes (valid_inter_S).
#define CUDANP_DISPATCH_S_INTER(S, ...)                  \
  switch (S) {                                           \
    case 3: { constexpr int kS = 3; __VA_ARGS__; } break;   \
    case 5: { constexpr int kS = 5; __VA_ARGS__; } break;   \
    case 10: { constexpr int kS = 10; __VA_ARGS__; } break; \
    case 15: { constexpr int kS = 15; __VA_ARGS__; } break; \
    default: return fail_invalid("inter-warp S must be one of 1..32 listed in cudanp.h"); \
  }
