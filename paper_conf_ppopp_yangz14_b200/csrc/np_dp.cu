// np_dp.cu -- the dynamic-parallelism comparison kernels (CDP2).
//
// The paper's alternative to CUDA-NP: a parent
// thread launches a child grid for its parallel loop through the device
// runtime; parent and child communicate through global memory only.  Two
// granularities, as in P:482:
//   per-thread: every master launches one child for its own loop;
//   per-block : the first thread of each CTA launches one child grid that
//               covers all the CTA's masters (the paper's manual fix for NN).
// CDP2 (CUDA 12) has no device-side synchronisation, so the child stores the
// item's result itself (R20).  This translation unit alone is built
// with -rdc=true; the NP kernels are not, so they carry no
// "dynamic-parallelism-enabled kernel overhead".
//
// A child launch the device runtime refuses (e.g. the pending-launch limit)
// increments g_dp_errors instead of failing silently.
#include "common.cuh"
#include "np_team.cuh"

namespace cudanp {

__device__ unsigned long long g_dp_errors = 0;

constexpr int kChildMax = 256;

__device__ __forceinline__ void note_launch() {
  if (cudaGetLastError() != cudaSuccess) atomicAdd(&g_dp_errors, 1ull);
}

// Block-wide fold of one value per thread (blockDim.x <= 1024, multiple of 32).
template <class T, class Op>
__device__ __forceinline__ T block_fold(T v, T* sh /*[32]*/) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = Op::apply(v, __shfl_xor_sync(kFull, v, o));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
  if (lane == 0) sh[warp] = v;
  __syncthreads();
  T r = sh[0];
  for (int k = 1; k < nw; ++k) r = Op::apply(r, sh[k]);
  __syncthreads();
  return r;
}

// Block-wide inclusive scan of one value per thread; *total = block sum.
template <class T>
__device__ __forceinline__ T block_scan(T v, T* sh /*[32]*/, T* total) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T t = __shfl_up_sync(kFull, v, o);
    if (lane >= o) v = OpSum::apply(v, t);
  }
  if (lane == 31) sh[warp] = v;
  __syncthreads();
  T off = T(0), all = T(0);
  for (int k = 0; k < nw; ++k) {
    if (k < warp) off = OpSum::apply(off, sh[k]);
    all = OpSum::apply(all, sh[k]);
  }
  __syncthreads();
  *total = all;
  return OpSum::apply(off, v);
}

__host__ __device__ inline int child_threads(int64_t L) {
  int64_t t = (L + 31) / 32 * 32;
  if (t < 32) t = 32;
  return (int)(t < kChildMax ? t : kChildMax);
}

// ---------------------------------------------------------------- children
// Child grid: blockIdx.x selects the master (item0 + blockIdx.x); its threads
// run the loop cyclically and fold the partials.
__global__ void dp_tmv_child(const float* A, int64_t lda, const float* x, float* y, int64_t col0,
                             int64_t ncols, int64_t h) {
  __shared__ float sh[32];
  const int64_t j = col0 + blockIdx.x;
  float acc = 0.f;
  for (int64_t i = threadIdx.x; i < h; i += blockDim.x) acc = fmaf(A[i * lda + j], x[i], acc);
  acc = block_fold<float, OpSum>(acc, sh);
  if (threadIdx.x == 0) y[j] = acc;
}

__global__ void dp_mv_child(const float* A, int64_t lda, const float* x, float* y, int64_t row0,
                            int64_t nrows, int64_t w) {
  __shared__ float sh[32];
  const int64_t i = row0 + blockIdx.x;
  float acc = 0.f;
  for (int64_t j = threadIdx.x; j < w; j += blockDim.x) acc = fmaf(A[i * lda + j], x[j], acc);
  acc = block_fold<float, OpSum>(acc, sh);
  if (threadIdx.x == 0) y[i] = acc;
}

template <class T, class Op>
__global__ void dp_reduce_child(const T* in, const T* init, T* out, int64_t item0, int64_t L) {
  __shared__ T sh[32];
  const int64_t n = item0 + blockIdx.x;
  T acc = Op::template identity<T>();
  for (int64_t i = threadIdx.x; i < L; i += blockDim.x) acc = Op::apply(acc, in[n * L + i]);
  acc = block_fold<T, Op>(acc, sh);
  if (threadIdx.x == 0) out[n] = init ? Op::apply(init[n], acc) : acc;
}

template <class T>
__global__ void dp_scan_child(const T* in, const T* init, T* out, int64_t item0, int64_t L) {
  __shared__ T sh[32];
  const int64_t n = item0 + blockIdx.x;
  T carry = init ? init[n] : T(0);
  for (int64_t base = 0; base < L; base += blockDim.x) {
    const int64_t i = base + threadIdx.x;
    const T v = i < L ? in[n * L + i] : T(0);
    T total;
    const T incl = block_scan<T>(v, sh, &total);
    if (i < L) out[n * L + i] = OpSum::apply(carry, incl);
    carry = OpSum::apply(carry, total);
  }
}

// ---------------------------------------------------------------- parents
// PER_BLOCK = false: each thread launches a child for its own item;
// PER_BLOCK = true : thread 0 of each CTA launches one child grid for the
// CTA's blockDim.x items.
template <bool PER_BLOCK>
__global__ void dp_tmv_parent(const float* A, int64_t lda, const float* x, float* y, int64_t w,
                              int64_t h) {
  const int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int ct = child_threads(h);
  if (PER_BLOCK) {
    if (threadIdx.x != 0) return;
    const int64_t c0 = (int64_t)blockIdx.x * blockDim.x;
    const int64_t nc = w - c0 < blockDim.x ? w - c0 : blockDim.x;
    dp_tmv_child<<<(unsigned)nc, ct, 0, cudaStreamFireAndForget>>>(A, lda, x, y, c0, nc, h);
    note_launch();
  } else {
    if (j >= w) return;
    dp_tmv_child<<<1, ct, 0, cudaStreamFireAndForget>>>(A, lda, x, y, j, 1, h);
    note_launch();
  }
}

template <bool PER_BLOCK>
__global__ void dp_mv_parent(const float* A, int64_t lda, const float* x, float* y, int64_t h,
                             int64_t w) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int ct = child_threads(w);
  if (PER_BLOCK) {
    if (threadIdx.x != 0) return;
    const int64_t r0 = (int64_t)blockIdx.x * blockDim.x;
    const int64_t nr = h - r0 < blockDim.x ? h - r0 : blockDim.x;
    dp_mv_child<<<(unsigned)nr, ct, 0, cudaStreamFireAndForget>>>(A, lda, x, y, r0, nr, w);
    note_launch();
  } else {
    if (i >= h) return;
    dp_mv_child<<<1, ct, 0, cudaStreamFireAndForget>>>(A, lda, x, y, i, 1, w);
    note_launch();
  }
}

template <class T, class Op, bool PER_BLOCK>
__global__ void dp_reduce_parent(const T* in, const T* init, T* out, int64_t N, int64_t L) {
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int ct = child_threads(L);
  if (PER_BLOCK) {
    if (threadIdx.x != 0) return;
    const int64_t n0 = (int64_t)blockIdx.x * blockDim.x;
    const int64_t nn = N - n0 < blockDim.x ? N - n0 : blockDim.x;
    dp_reduce_child<T, Op><<<(unsigned)nn, ct, 0, cudaStreamFireAndForget>>>(in, init, out, n0, L);
    note_launch();
  } else {
    if (n >= N) return;
    dp_reduce_child<T, Op><<<1, ct, 0, cudaStreamFireAndForget>>>(in, init, out, n, L);
    note_launch();
  }
}

template <class T, bool PER_BLOCK>
__global__ void dp_scan_parent(const T* in, const T* init, T* out, int64_t N, int64_t L) {
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int ct = child_threads(L);
  if (PER_BLOCK) {
    if (threadIdx.x != 0) return;
    const int64_t n0 = (int64_t)blockIdx.x * blockDim.x;
    const int64_t nn = N - n0 < blockDim.x ? N - n0 : blockDim.x;
    dp_scan_child<T><<<(unsigned)nn, ct, 0, cudaStreamFireAndForget>>>(in, init, out, n0, L);
    note_launch();
  } else {
    if (n >= N) return;
    dp_scan_child<T><<<1, ct, 0, cudaStreamFireAndForget>>>(in, init, out, n, L);
    note_launch();
  }
}

// ---------------------------------------------------------------- memcopy microbenchmark (Fig 1)
// copy m*n floats; the parent kernel has m threads and each launches
// a child grid of n threads that copies n floats.  memcopy_rdc_kernel is the
// plain copy compiled inside this -rdc translation unit, i.e. the "dynamic-
// parallelism-enabled kernel overhead" case; the same kernel without
// -rdc lives in abi.cu.
__global__ void memcopy_rdc_kernel(const float* __restrict__ in, float* __restrict__ out,
                                   int64_t total) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
       i += (int64_t)gridDim.x * blockDim.x)
    out[i] = in[i];
}

__global__ void dp_memcopy_child(const float* __restrict__ in, float* __restrict__ out, int64_t n) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) out[i] = in[i];
}

__global__ void dp_memcopy_parent(const float* in, float* out, int64_t m, int64_t n) {
  const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= m) return;
  const int64_t base = p * n;
  const unsigned blocks = (unsigned)((n + 255) / 256);
  dp_memcopy_child<<<blocks, n < 256 ? (unsigned)((n + 31) / 32 * 32) : 256u, 0,
                     cudaStreamFireAndForget>>>(in + base, out + base, n);
  note_launch();
}

int dp_memcopy(const float* in, float* out, int64_t total, int64_t m, int variant, cudaStream_t st) {
  if (total == 0) return CUDANP_OK;
  if (variant == 1) {
    memcopy_rdc_kernel<<<(unsigned)(sm_count() * 8), 256, 0, st>>>(in, out, total);
  } else {
    dp_memcopy_parent<<<(unsigned)((m + 127) / 128), 128, 0, st>>>(in, out, m, total / m);
  }
  return check_launch("dp_memcopy launch");
}

// ---------------------------------------------------------------- host side
constexpr int kParentBlock = 128;

static unsigned parent_grid(int64_t n) { return (unsigned)((n + kParentBlock - 1) / kParentBlock); }

int dp_tmv(bool per_block, const float* A, int64_t lda, const float* x, float* y, int64_t w,
           int64_t h, cudaStream_t st) {
  if (w == 0) return CUDANP_OK;
  if (per_block) dp_tmv_parent<true><<<parent_grid(w), kParentBlock, 0, st>>>(A, lda, x, y, w, h);
  else dp_tmv_parent<false><<<parent_grid(w), kParentBlock, 0, st>>>(A, lda, x, y, w, h);
  return check_launch("tmv dp launch");
}

int dp_mv(bool per_block, const float* A, int64_t lda, const float* x, float* y, int64_t h,
          int64_t w, cudaStream_t st) {
  if (h == 0) return CUDANP_OK;
  if (per_block) dp_mv_parent<true><<<parent_grid(h), kParentBlock, 0, st>>>(A, lda, x, y, h, w);
  else dp_mv_parent<false><<<parent_grid(h), kParentBlock, 0, st>>>(A, lda, x, y, h, w);
  return check_launch("mv dp launch");
}

template <class T, class Op>
static void launch_dp_reduce(bool pb, const void* in, const void* init, void* out, int64_t N,
                             int64_t L, cudaStream_t st) {
  if (pb)
    dp_reduce_parent<T, Op, true><<<parent_grid(N), kParentBlock, 0, st>>>((const T*)in, (const T*)init, (T*)out, N, L);
  else
    dp_reduce_parent<T, Op, false><<<parent_grid(N), kParentBlock, 0, st>>>((const T*)in, (const T*)init, (T*)out, N, L);
}

int dp_reduce(bool per_block, const void* in, const void* init, void* out, int64_t N, int64_t L,
              int dtype, int op, cudaStream_t st) {
  if (N == 0) return CUDANP_OK;
  if (dtype == CUDANP_F32) {
    if (op == CUDANP_SUM) launch_dp_reduce<float, OpSum>(per_block, in, init, out, N, L, st);
    else launch_dp_reduce<float, OpMax>(per_block, in, init, out, N, L, st);
  } else {
    if (op == CUDANP_SUM) launch_dp_reduce<int32_t, OpSum>(per_block, in, init, out, N, L, st);
    else launch_dp_reduce<int32_t, OpMax>(per_block, in, init, out, N, L, st);
  }
  return check_launch("batched_loop_reduce dp launch");
}

int dp_scan(bool per_block, const void* in, const void* init, void* out, int64_t N, int64_t L,
            int dtype, cudaStream_t st) {
  if (N == 0 || L == 0) return CUDANP_OK;
  if (dtype == CUDANP_F32) {
    if (per_block) dp_scan_parent<float, true><<<parent_grid(N), kParentBlock, 0, st>>>((const float*)in, (const float*)init, (float*)out, N, L);
    else dp_scan_parent<float, false><<<parent_grid(N), kParentBlock, 0, st>>>((const float*)in, (const float*)init, (float*)out, N, L);
  } else {
    if (per_block) dp_scan_parent<int32_t, true><<<parent_grid(N), kParentBlock, 0, st>>>((const int32_t*)in, (const int32_t*)init, (int32_t*)out, N, L);
    else dp_scan_parent<int32_t, false><<<parent_grid(N), kParentBlock, 0, st>>>((const int32_t*)in, (const int32_t*)init, (int32_t*)out, N, L);
  }
  return check_launch("batched_loop_scan dp launch");
}

int dp_error_count(int reset, int64_t* count) {
  unsigned long long c = 0;
  if (cudaDeviceSynchronize() != cudaSuccess ||
      cudaMemcpyFromSymbol(&c, g_dp_errors, sizeof(c)) != cudaSuccess) {
    return check_launch("dp_error_count");
  }
  if (count) *count = (int64_t)c;
  if (reset) {
    c = 0;
    if (cudaMemcpyToSymbol(g_dp_errors, &c, sizeof(c)) != cudaSuccess) return check_launch("dp_error_count reset");
  }
  return CUDANP_OK;
}

}  // namespace cudanp
