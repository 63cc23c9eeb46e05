// np_tmv_tma.cu -- TMV with TMA-staged tiles (the north star's "TMA or
// cp.async staging where the access pattern is strided (as in y=A^T x)").
//
// Same method as tmv_inter_kernel (Fig 2; inter-warp NP):
// a CTA owns COLS = 32 x V column-masters' outputs (V per lane) and S slave
// warps share the rows, cyclic or block (R5); the S partials meet in
// shared memory and the master warp stores.  What changes is
// how A reaches the slaves: instead of each lane issuing 128-bit loads, one
// elected thread streams [rows x COLS columns] tiles of A into a ring of
// shared-memory stages with the Tensor Memory Accelerator
// (cp.async.bulk.tensor.2d, completion counted on an mbarrier), and the
// slaves read their rows from shared memory.  Memory-level parallelism then
// comes from the stages in flight, not from the number of resident threads.
//
//  cyclic: one box of R rows per stage (TmaShape); slave s owns the box rows
//          k*S + s, i.e. global rows i = s (mod S) exactly as P:166.
//  block : S boxes of R/S rows per stage, one from each slave's contiguous
//          chunk [s*c, (s+1)*c) (c = ceil(h/S)).
// Rows past h come back zero-filled by TMA and are masked before x is read.
#include <cuda.h>

#include "common.cuh"
#include "np_team.cuh"

namespace cudanp {

// Rows per stage and ring depth per S.  Every consumer warp spins on the
// stage's mbarrier, so stages must carry enough rows per slave to amortise
// the waits (measured on C2: 32 rows x 8 stages is best for S <= 2, 128 x 4
// for S = 4, 256 x 4 for S >= 8; box height <= 256).
template <int S> struct TmaShape {
  static constexpr int ROWS = S <= 2 ? 32 : (S == 4 ? 128 : 256);
  static constexpr int STAGES = S <= 2 ? 8 : 4;
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n"
      "WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}" ::"r"(smem_u32(b)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, int c0, int c1,
                                            uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3}], [%4];" ::"r"(smem_u32(dst)),
      "l"((uint64_t)map), "r"(c0), "r"(c1), "r"(smem_u32(bar))
      : "memory");
}

// COLS = columns per CTA = 32 lanes x V (V = 4, 2, 1): narrower CTAs give
// more of them, so C2's 16384 columns cover every SM several times.
template <int S, int DIST, int COLS>
__global__ void __launch_bounds__(32 * S)
tmv_tma_kernel(const __grid_constant__ CUtensorMap mapA, const float* __restrict__ x,
               float* __restrict__ y, int64_t w, int64_t h) {
  constexpr int kTmaCols = COLS;
  constexpr int V = COLS / 32;
  constexpr int R = TmaShape<S>::ROWS;
  constexpr int kTmaStages = TmaShape<S>::STAGES;
  constexpr int RK = R / S;  // rows per slave per stage
  static_assert(R % S == 0, "S must divide the rows per stage");
  extern __shared__ __align__(128) unsigned char smem_raw[];
  float* tiles = reinterpret_cast<float*>(smem_raw);                   // [stages][R][128]
  uint64_t* full = reinterpret_cast<uint64_t*>(tiles + kTmaStages * R * kTmaCols);
  uint64_t* empty = full + kTmaStages;
  float* red = reinterpret_cast<float*>(empty + kTmaStages);          // [S][128]

  const int lane = threadIdx.x & 31, s = threadIdx.x >> 5;            // master lane, slave warp
  const int col0 = blockIdx.x * kTmaCols;
  const int64_t c = (h + S - 1) / S;                                  // block: rows per chunk
  const int64_t per_slave = DIST == DIST_CYCLIC ? (h + S - 1) / S : c;
  const int ntiles = (int)((per_slave + RK - 1) / RK);
  const bool producer = threadIdx.x == 0;

  if (producer) {
    for (int i = 0; i < kTmaStages; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], S);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  auto issue = [&](int t) {
    const int st = t % kTmaStages;
    float* dst = tiles + st * R * kTmaCols;
    mbar_expect_tx(&full[st], R * kTmaCols * 4);
    if (DIST == DIST_CYCLIC) {
      tma_load_2d(dst, &mapA, col0, t * R, &full[st]);
    } else {
      for (int k = 0; k < S; ++k)
        tma_load_2d(dst + k * RK * kTmaCols, &mapA, col0, (int)(k * c + (int64_t)t * RK), &full[st]);
    }
  };
  if (producer)
    for (int t = 0; t < kTmaStages && t < ntiles; ++t) issue(t);

  V4<float> acc = {0.f, 0.f, 0.f, 0.f};
  for (int t = 0; t < ntiles; ++t) {
    const int st = t % kTmaStages;
    const uint32_t par = (t / kTmaStages) & 1;
    // x does not depend on the TMA: issue its loads before waiting on the
    // stage so their latency hides behind the tile's arrival.
    float xs[RK];
#pragma unroll
    for (int kk = 0; kk < RK; ++kk) {
      int64_t row;
      bool ok;
      if (DIST == DIST_CYCLIC) {
        row = (int64_t)t * R + kk * S + s;
        ok = row < h;
      } else {
        const int64_t k = (int64_t)t * RK + kk;
        row = s * c + k;
        ok = k < c && row < h;
      }
      xs[kk] = ok ? __ldg(x + row) : 0.f;
    }
    mbar_wait(&full[st], par);
    const float* tile = tiles + st * R * kTmaCols;
#pragma unroll
    for (int kk = 0; kk < RK; ++kk) {
      const int lr = DIST == DIST_CYCLIC ? kk * S + s : s * RK + kk;
      const float xv = xs[kk];
      const float* ap = tile + lr * kTmaCols + lane * V;
      if constexpr (V == 4) {
        const float4 a = *reinterpret_cast<const float4*>(ap);
        acc.x = fmaf(a.x, xv, acc.x); acc.y = fmaf(a.y, xv, acc.y);
        acc.z = fmaf(a.z, xv, acc.z); acc.w = fmaf(a.w, xv, acc.w);
      } else if constexpr (V == 2) {
        const float2 a = *reinterpret_cast<const float2*>(ap);
        acc.x = fmaf(a.x, xv, acc.x); acc.y = fmaf(a.y, xv, acc.y);
      } else {
        acc.x = fmaf(*ap, xv, acc.x);
      }
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[st]);      // this slave is done with the stage
    if (producer && t + kTmaStages < ntiles) {
      mbar_wait(&empty[st], par);                 // every slave released it
      issue(t + kTmaStages);
    }
  }
  // team reduction through shared memory; the master warp folds in slave order
  float* rr = red + s * kTmaCols + lane * V;
  const float av[4] = {acc.x, acc.y, acc.z, acc.w};
#pragma unroll
  for (int v = 0; v < V; ++v) rr[v] = av[v];
  __syncthreads();
  if (s == 0) {
    const int64_t col = col0 + lane * V;
    float sum[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
    for (int k = 0; k < S; ++k) {
      const float* p = red + k * kTmaCols + lane * V;
#pragma unroll
      for (int v = 0; v < V; ++v) sum[v] += p[v];
    }
#pragma unroll
    for (int v = 0; v < V; ++v)
      if (col + v < w) y[col + v] = sum[v];
  }
}

// ---------------------------------------------------------------- host side
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess)
      fn = (EncodeTiledFn)f;
    else
      cudaGetLastError();
  }
  return fn;
}

template <int S, int DIST, int kTmaCols>
static int launch_tmv_tma_s(const float* A, int64_t lda, const float* x, float* y, int64_t w,
                            int64_t h, cudaStream_t st) {
  EncodeTiledFn enc = encode_fn();
  if (!enc) {
    set_error("cuTensorMapEncodeTiled entry point unavailable");
    return CUDANP_ERR_CUDA;
  }
  CUtensorMap map;
  const cuuint64_t dims[2] = {(cuuint64_t)w, (cuuint64_t)h};
  const cuuint64_t strides[1] = {(cuuint64_t)lda * 4};
  constexpr int kTmaRows = TmaShape<S>::ROWS, kTmaStages = TmaShape<S>::STAGES;
  const cuuint32_t box[2] = {kTmaCols, DIST == DIST_CYCLIC ? (cuuint32_t)kTmaRows : (cuuint32_t)(kTmaRows / S)};
  const cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void*)A, dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    set_error("cuTensorMapEncodeTiled failed (%d)", (int)r);
    return CUDANP_ERR_CUDA;
  }
  const size_t smem = (size_t)kTmaStages * kTmaRows * kTmaCols * 4 + 2 * kTmaStages * 8 +
                      (size_t)S * kTmaCols * 4;
  auto kern = tmv_tma_kernel<S, DIST, kTmaCols>;
  if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return check_launch("tmv_tma smem attribute");
  const unsigned grid = (unsigned)((w + kTmaCols - 1) / kTmaCols);
  kern<<<grid, 32 * S, smem, st>>>(map, x, y, w, h);
  return check_launch("tmv_tma launch");
}

// Preconditions (checked by the ABI): A 16-byte aligned, lda % 4 == 0,
// h and w < 2^31 (TMA coordinates are int32).
int tmv_tma(const float* A, int64_t lda, const float* x, float* y, int64_t w, int64_t h, int S,
            int dist, cudaStream_t st) {
  if (w == 0) return CUDANP_OK;
  // CTA width: the widest of 128/64/32 columns that still gives >= 2 CTAs per SM.
  const int sms = sm_count();
  const int cols = (w + 127) / 128 >= 2 * sms ? 128 : ((w + 63) / 64 >= 2 * sms ? 64 : 32);
  CUDANP_DISPATCH_S(S, {
    if (cols == 128)
      return dist == DIST_CYCLIC ? launch_tmv_tma_s<kS, DIST_CYCLIC, 128>(A, lda, x, y, w, h, st)
                                 : launch_tmv_tma_s<kS, DIST_BLOCK, 128>(A, lda, x, y, w, h, st);
    if (cols == 64)
      return dist == DIST_CYCLIC ? launch_tmv_tma_s<kS, DIST_CYCLIC, 64>(A, lda, x, y, w, h, st)
                                 : launch_tmv_tma_s<kS, DIST_BLOCK, 64>(A, lda, x, y, w, h, st);
    return dist == DIST_CYCLIC ? launch_tmv_tma_s<kS, DIST_CYCLIC, 32>(A, lda, x, y, w, h, st)
                               : launch_tmv_tma_s<kS, DIST_BLOCK, 32>(A, lda, x, y, w, h, st);
  });
  return CUDANP_OK;
}

}  // namespace cudanp
