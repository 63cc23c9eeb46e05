// np_s1_tiled.cu -- the no-NP (S = 1) baselines whose rows reach the thread
// through shared-memory tiles, for MV and the batched scan.
//
// The paper's speedups are over "already optimized" kernels:
// its MV baseline is the shared-memory-tiled SMM kernel (Table 1: the
// baseline MV uses 132 B of shared memory per thread), not a thread that walks
// its row with strided loads.  One thread per item reading its own row
// directly makes every warp load touch 32 different rows (32 sectors per
// request); the tiled form stages a [R rows x 32 columns] tile with a coalesced
// copy and lets each thread read its row out of shared memory.  On sm_100a the
// copy is a TMA 2-D box (cp.async.bulk.tensor) with the 128-byte swizzle, so
// the row-per-thread reads (LDS.128 of row r, chunk c at chunk c ^ (r & 7))
// are bank-conflict-free, and a ring of stages keeps the bytes in flight that
// 128 threads per SM could not.  These kernels are the S = 1 denominators of
// the NP speedups (CUDANP_IMPL_S1_TILED); the method (one master, no slaves)
// is the literal Fig 2 loop.
//
//  MV:   a CTA owns R rows; a producer warp streams the column tiles -- and
//        the matching 128-byte chunk of x, a 1-D tensor box on the same
//        barrier (zero-filled past w) -- into the ring; each consumer thread
//        accumulates its row (acc += A[r][j]*x[j], x read from shared memory
//        as a broadcast) and stores y[r].
//  reduce: the same walk; each thread folds its row's elements of every tile
//        (sum or max) and the master -- the thread itself -- applies init[n]
//        and stores out[n] at the row's last tile.
//  scan: a persistent CTA walks (row group, column tile) tiles; each thread
//        scans its row's 32 elements in place in shared memory with its
//        running carry (init[n] at the row's first tile), the CTA stores the
//        tile back with a TMA store, and the stage is refilled once the store
//        has read it (bulk-group wait).
#include <cuda.h>

#include "common.cuh"
#include "np_team.cuh"
#include "np_tma.cuh"

namespace cudanp {

constexpr int kS1Cols = 32;  // tile width: 32 x 4 B = one 128-byte swizzle row

// Element offset of float4 chunk c (0..7) of row r in a SWIZZLE_128B tile.
__device__ __forceinline__ int swz128(int r, int c) { return r * kS1Cols + ((c ^ (r & 7)) << 2); }

__device__ __forceinline__ void tma_load_1d(void* dst, const CUtensorMap* map, int c0, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.1d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2}], [%3];" ::"r"(smem_u32(dst)),
      "l"((uint64_t)map), "r"(c0), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* map, int c0, int c1, const void* src) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];" ::"l"(
                   (uint64_t)map),
               "r"(c0), "r"(c1), "r"(smem_u32(src))
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// 1 KB header (mbarriers), then 1024-byte aligned stages (the 128-byte
// swizzle repeats every 8 rows = 1 KB, and TMA wants the box base aligned).
constexpr size_t kS1Header = 1024;

// ---------------------------------------------------------------- MV, S = 1
template <int R>
__global__ void __launch_bounds__(R + 32, 1)
mv_s1_tiled_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapX,
                   float* __restrict__ y, int64_t h, int64_t w, int stages) {
  pdl_entry();
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  unsigned char* base = smem_raw + ((1024 - (smem_u32(smem_raw) & 1023)) & 1023);
  uint64_t* full = reinterpret_cast<uint64_t*>(base);   // A tile and x chunk landed
  uint64_t* empty = full + stages;                         // consumers done with the stage
  float* tiles = reinterpret_cast<float*>(base + kS1Header);
  float* xs = tiles + stages * (R * kS1Cols);              // [stages][32]
  constexpr int kWarps = R / 32;
  constexpr uint32_t kStageBytes = R * kS1Cols * 4;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int row0 = blockIdx.x * R;
  const int ntiles = (int)((w + kS1Cols - 1) / kS1Cols);

  if (threadIdx.x == 0) {
    for (int i = 0; i < stages; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], kWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  if (warp == kWarps) {  // producer warp
    if (lane == 0) {
      for (int t = 0; t < ntiles; ++t) {
        const int st = t % stages;
        if (t >= stages) mbar_wait(&empty[st], ((t / stages) - 1) & 1);
        mbar_expect_tx(&full[st], kStageBytes + kS1Cols * 4);
        tma_load_2d(tiles + st * (R * kS1Cols), &mapA, t * kS1Cols, row0, &full[st]);
        tma_load_1d(xs + st * kS1Cols, &mapX, t * kS1Cols, &full[st]);
      }
    }
    return;
  }
  const int r = threadIdx.x;
  V4<float> acc = {0.f, 0.f, 0.f, 0.f};
  for (int t = 0; t < ntiles; ++t) {
    const int st = t % stages;
    mbar_wait(&full[st], (t / stages) & 1);
    const float* tile = tiles + st * (R * kS1Cols);
    const float* xt = xs + st * kS1Cols;
#pragma unroll
    for (int c = 0; c < 8; ++c) {  // (past w both the tile and the x chunk are zero-filled)
      const float4 a = *reinterpret_cast<const float4*>(tile + swz128(r, c));
      const float4 xv = *reinterpret_cast<const float4*>(xt + 4 * c);  // broadcast
      acc.x = fmaf(a.x, xv.x, acc.x); acc.y = fmaf(a.y, xv.y, acc.y);
      acc.z = fmaf(a.z, xv.z, acc.z); acc.w = fmaf(a.w, xv.w, acc.w);
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[st]);
  }
  if (row0 + r < h) y[row0 + r] = (acc.x + acc.y) + (acc.z + acc.w);
}

// ---------------------------------------------------------------- scan, S = 1
template <class T, int R>
__global__ void __launch_bounds__(R, 1)
scan_s1_tiled_kernel(const __grid_constant__ CUtensorMap mapIn, const __grid_constant__ CUtensorMap mapOut,
                     const T* __restrict__ init, int64_t N, int64_t L, int stages) {
  pdl_entry();
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  unsigned char* base = smem_raw + ((1024 - (smem_u32(smem_raw) & 1023)) & 1023);
  uint64_t* full = reinterpret_cast<uint64_t*>(base);
  T* tiles = reinterpret_cast<T*>(base + kS1Header);
  constexpr uint32_t kStageBytes = R * kS1Cols * 4;
  const int r = threadIdx.x;
  const int64_t ngroups = (N + R - 1) / R;
  const int nk = (int)((L + kS1Cols - 1) / kS1Cols);
  const int64_t mygroups = blockIdx.x < ngroups ? (ngroups - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  const int64_t ntiles = mygroups * nk;
  auto coords = [&](int64_t t, int& col, int& row) {
    const int64_t g = blockIdx.x + (t / nk) * gridDim.x;
    col = (int)(t % nk) * kS1Cols;
    row = (int)(g * R);
  };
  if (r == 0) {
    for (int i = 0; i < stages; ++i) mbar_init(&full[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    for (int64_t t = 0; t < stages - 1 && t < ntiles; ++t) {  // prologue: stages-1 tiles ahead
      int col, row;
      coords(t, col, row);
      mbar_expect_tx(&full[t], kStageBytes);
      tma_load_2d(tiles + t * (R * kS1Cols), &mapIn, col, row, &full[t]);
    }
  }
  __syncthreads();
  T carry = T(0);
  for (int64_t t = 0; t < ntiles; ++t) {
    const int st = (int)(t % stages);
    int col, row;
    coords(t, col, row);
    if (col == 0) {  // the item's sequential section: its carry-in
      const int64_t n = (int64_t)row + r;
      carry = (init && n < N) ? init[n] : T(0);
    }
    mbar_wait(&full[st], (uint32_t)(t / stages) & 1);
    T* tile = tiles + st * (R * kS1Cols);
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      V4<T>* p = reinterpret_cast<V4<T>*>(tile + swz128(r, c));
      V4<T> v = *p;
      v.x = OpSum::apply(carry, v.x); v.y = OpSum::apply(v.x, v.y);
      v.z = OpSum::apply(v.y, v.z); v.w = OpSum::apply(v.z, v.w);
      carry = v.w;
      *p = v;
    }
    fence_proxy_async_smem();  // the threads' writes, visible to the TMA store
    __syncthreads();
    if (r == 0) {
      tma_store_2d(&mapOut, col, row, tile);  // clipped to [N) x [L) by the tensor map
      bulk_commit();
      const int64_t tn = t + stages - 1;      // refill the stage of tile t-1 ...
      if (tn < ntiles) {
        bulk_wait_read<1>();                  // ... once its store has read it
        int c2, r2;
        coords(tn, c2, r2);
        const int sn = (int)(tn % stages);
        mbar_expect_tx(&full[sn], kStageBytes);
        tma_load_2d(tiles + sn * (R * kS1Cols), &mapIn, c2, r2, &full[sn]);
      }
    }
  }
  if (r == 0) bulk_wait_all();  // stores done before the CTA's shared memory goes away
}

// ---------------------------------------------------------------- reduce, S = 1
// Stage s is refilled (tile t + stages) once every thread has passed tile t's
// barrier; columns past L (zero-filled by TMA) are skipped, so max sees only
// the row's own elements.
template <class T, class Op, int R>
__global__ void __launch_bounds__(R, 1)
reduce_s1_tiled_kernel(const __grid_constant__ CUtensorMap mapIn, const T* __restrict__ init,
                       T* __restrict__ out, int64_t N, int64_t L, int stages) {
  pdl_entry();
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  unsigned char* base = smem_raw + ((1024 - (smem_u32(smem_raw) & 1023)) & 1023);
  uint64_t* full = reinterpret_cast<uint64_t*>(base);
  const T* tiles = reinterpret_cast<const T*>(base + kS1Header);
  constexpr uint32_t kStageBytes = R * kS1Cols * 4;
  const int r = threadIdx.x;
  const int64_t ngroups = (N + R - 1) / R;
  const int nk = (int)((L + kS1Cols - 1) / kS1Cols);
  const int64_t mygroups = blockIdx.x < ngroups ? (ngroups - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  const int64_t ntiles = mygroups * nk;
  auto coords = [&](int64_t t, int& col, int& row) {
    const int64_t g = blockIdx.x + (t / nk) * gridDim.x;
    col = (int)(t % nk) * kS1Cols;
    row = (int)(g * R);
  };
  if (r == 0) {
    for (int i = 0; i < stages; ++i) mbar_init(&full[i], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    for (int64_t t = 0; t < stages && t < ntiles; ++t) {
      int col, row;
      coords(t, col, row);
      mbar_expect_tx(&full[t], kStageBytes);
      tma_load_2d(const_cast<T*>(tiles) + t * (R * kS1Cols), &mapIn, col, row, &full[t]);
    }
  }
  __syncthreads();
  const T id = Op::template identity<T>();
  T acc = id;
  for (int64_t t = 0; t < ntiles; ++t) {
    const int st = (int)(t % stages);
    int col, row;
    coords(t, col, row);
    mbar_wait(&full[st], (uint32_t)(t / stages) & 1);
    const T* tile = tiles + st * (R * kS1Cols);
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      if (col + 4 * c >= L) break;
      const V4<T> v = *reinterpret_cast<const V4<T>*>(tile + swz128(r, c));
      acc = Op::apply(acc, Op::apply(Op::apply(v.x, v.y), Op::apply(v.z, v.w)));
    }
    if (col + kS1Cols >= L) {  // the row's last tile: the master finishes the item
      const int64_t n = (int64_t)row + r;
      if (n < N) out[n] = init ? Op::apply(init[n], acc) : acc;
      acc = id;
    }
    __syncthreads();  // every thread is done with stage st
    if (r == 0 && t + stages < ntiles) {
      int c2, r2;
      coords(t + stages, c2, r2);
      mbar_expect_tx(&full[st], kStageBytes);
      tma_load_2d(const_cast<T*>(tiles) + st * (R * kS1Cols), &mapIn, c2, r2, &full[st]);
    }
  }
}

// ---------------------------------------------------------------- host side
typedef CUresult (*EncodeTiledFnS1)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                    const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                    const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                    CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFnS1 encode_fn_s1() {
  static EncodeTiledFnS1 fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess)
      fn = (EncodeTiledFnS1)f;
    else
      cudaGetLastError();
  }
  return fn;
}

// rows x cols 4-byte elements, row pitch ld elements, box [32 cols x box_rows], 128-byte swizzle
static int encode_s1(CUtensorMap* map, const void* p, int64_t rows, int64_t cols, int64_t ld,
                     int box_rows) {
  EncodeTiledFnS1 enc = encode_fn_s1();
  if (!enc) {
    set_error("cuTensorMapEncodeTiled entry point unavailable");
    return CUDANP_ERR_CUDA;
  }
  const cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  const cuuint64_t strides[1] = {(cuuint64_t)ld * 4};
  const cuuint32_t box[2] = {(cuuint32_t)kS1Cols, (cuuint32_t)box_rows};
  const cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<void*>(p), dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    set_error("cuTensorMapEncodeTiled failed (%d)", (int)r);
    return CUDANP_ERR_CUDA;
  }
  return CUDANP_OK;
}

// x as a 1-D tensor of w floats, box of 32 (one 128-byte chunk per stage).
static int encode_x1(CUtensorMap* map, const float* x, int64_t w) {
  EncodeTiledFnS1 enc = encode_fn_s1();
  if (!enc) {
    set_error("cuTensorMapEncodeTiled entry point unavailable");
    return CUDANP_ERR_CUDA;
  }
  const cuuint64_t dims[1] = {(cuuint64_t)w};
  const cuuint64_t strides[1] = {0};
  const cuuint32_t box[1] = {(cuuint32_t)kS1Cols};
  const cuuint32_t estr[1] = {1};
  CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 1, const_cast<float*>(x), dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                   CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    set_error("cuTensorMapEncodeTiled (x) failed (%d)", (int)r);
    return CUDANP_ERR_CUDA;
  }
  return CUDANP_OK;
}

// Ring depth for `per_sm` resident CTAs of `stage` bytes (<= 227 KB per CTA,
// 228 KB per SM, 1 KB reserved per CTA), at most 12 stages.
static int s1_stages(int per_sm, size_t stage) {
  size_t budget = (228 * 1024) / (size_t)per_sm;
  budget = budget > 1024 + kS1Header + 1024 ? budget - 1024 - kS1Header - 1024 : 0;
  if (budget > 227 * 1024 - kS1Header - 1024) budget = 227 * 1024 - kS1Header - 1024;
  int s = (int)(budget / stage);
  return s < 2 ? 2 : (s > 12 ? 12 : s);
}

template <int R>
static int launch_mv_s1(const float* A, int64_t lda, const float* x, float* y, int64_t h, int64_t w,
                        cudaStream_t st) {
  CUtensorMap map, mapx;
  if (int rc = encode_s1(&map, A, h, w, lda, R)) return rc;
  if (int rc = encode_x1(&mapx, x, w)) return rc;
  const int64_t grid = (h + R - 1) / R;
  const int sms = sm_count();
  const int per_sm = (int)((grid + sms - 1) / sms) < 2 ? 1 : 2;
  const int stages = s1_stages(per_sm, (size_t)R * kS1Cols * 4 + kS1Cols * 4);
  const size_t smem = kS1Header + 1024 + (size_t)stages * (R * kS1Cols * 4 + kS1Cols * 4);
  auto kern = mv_s1_tiled_kernel<R>;
  if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return check_launch("mv S=1 tiled smem attribute");
  launch_pdl(kern, dim3((unsigned)grid), dim3(R + 32), smem, st, map, mapx, y, h, w, stages);
  return check_launch("mv S=1 tiled launch");
}

// y = A x with one thread per row, rows staged by TMA (needs A 16-byte
// aligned, lda % 4 == 0, sizes < 2^31; the ABI checks).  128-row CTAs when
// they give every SM one, else 64-row CTAs.
int mv_s1_tiled(const float* A, int64_t lda, const float* x, float* y, int64_t h, int64_t w,
                cudaStream_t st) {
  if (h == 0) return CUDANP_OK;
  if (w == 0) {
    if (cudaMemsetAsync(y, 0, (size_t)h * 4, st) != cudaSuccess) return check_launch("mv S=1 zero");
    return CUDANP_OK;
  }
  if ((h + 127) / 128 >= sm_count()) return launch_mv_s1<128>(A, lda, x, y, h, w, st);
  return launch_mv_s1<64>(A, lda, x, y, h, w, st);
}

template <class T>
static int launch_scan_s1(const T* in, const T* init, T* out, int64_t N, int64_t L, cudaStream_t st) {
  constexpr int R = 128;
  CUtensorMap mi, mo;
  if (int rc = encode_s1(&mi, in, N, L, L, R)) return rc;
  if (int rc = encode_s1(&mo, out, N, L, L, R)) return rc;
  constexpr int kPerSM = 2;
  const int stages = s1_stages(kPerSM, (size_t)R * kS1Cols * 4);
  const size_t smem = kS1Header + 1024 + (size_t)stages * R * kS1Cols * 4;
  auto kern = scan_s1_tiled_kernel<T, R>;
  if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return check_launch("scan S=1 tiled smem attribute");
  const int64_t groups = (N + R - 1) / R;
  const int64_t grid = persistent_grid(kern, R, smem, groups);
  launch_pdl(kern, dim3((unsigned)grid), dim3(R), smem, st, mi, mo, init, N, L, stages);
  return check_launch("scan S=1 tiled launch");
}

template <class T, class Op>
static int launch_reduce_s1(const T* in, const T* init, T* out, int64_t N, int64_t L, cudaStream_t st) {
  constexpr int R = 128;
  CUtensorMap mi;
  if (int rc = encode_s1(&mi, in, N, L, L, R)) return rc;
  constexpr int kPerSM = 2;
  const int stages = s1_stages(kPerSM, (size_t)R * kS1Cols * 4);
  const size_t smem = kS1Header + 1024 + (size_t)stages * R * kS1Cols * 4;
  auto kern = reduce_s1_tiled_kernel<T, Op, R>;
  if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return check_launch("reduce S=1 tiled smem attribute");
  const int64_t grid = persistent_grid(kern, R, smem, (N + R - 1) / R);
  launch_pdl(kern, dim3((unsigned)grid), dim3(R), smem, st, mi, init, out, N, L, stages);
  return check_launch("reduce S=1 tiled launch");
}

// Loop-reduce with one thread per item, rows staged by TMA (needs `in`
// 16-byte aligned, L % 4 == 0, sizes < 2^31; the ABI checks).  L = 0 is the
// caller's (the NP path writes init / the identity).
int reduce_s1_tiled(const void* in, const void* init, void* out, int64_t N, int64_t L, int dtype,
                    int op, cudaStream_t st) {
  if (N == 0) return CUDANP_OK;
  if (dtype == CUDANP_F32)
    return op == CUDANP_SUM ? launch_reduce_s1<float, OpSum>((const float*)in, (const float*)init, (float*)out, N, L, st)
                            : launch_reduce_s1<float, OpMax>((const float*)in, (const float*)init, (float*)out, N, L, st);
  return op == CUDANP_SUM ? launch_reduce_s1<int32_t, OpSum>((const int32_t*)in, (const int32_t*)init, (int32_t*)out, N, L, st)
                          : launch_reduce_s1<int32_t, OpMax>((const int32_t*)in, (const int32_t*)init, (int32_t*)out, N, L, st);
}

// Inclusive scan with one thread per item, rows staged (and stored) by TMA
// (needs in/out 16-byte aligned, L % 4 == 0, sizes < 2^31; the ABI checks).
int scan_s1_tiled(const void* in, const void* init, void* out, int64_t N, int64_t L, int dtype,
                  cudaStream_t st) {
  if (N == 0 || L == 0) return CUDANP_OK;
  if (dtype == CUDANP_F32)
    return launch_scan_s1<float>((const float*)in, (const float*)init, (float*)out, N, L, st);
  return launch_scan_s1<int32_t>((const int32_t*)in, (const int32_t*)init, (int32_t*)out, N, L, st);
}

}  // namespace cudanp
