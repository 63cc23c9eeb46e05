// np_ragged.cu -- ragged (runtime-bounded) loop-reduce over CSR segments
// (SURVEY §8(f) row f1):  out[n] = init[n] (op) fold_{off[n] <= i < off[n+1]} in[i].
//
// This is the paper's runtime-bounded parallel loop in its plainest form:
// "as the loop bound checking remains in the transformed code, this
// transformation is valid if the loop bound is determined at the runtime"
// (P:193).  The bounds are live-ins computed by the master's sequential
// section (it loads off[n], off[n+1]) and handed to the slaves with
// read_from_master; the slaves share the loop (cyclic P:166 or
// block R5); the live-out is reduced and the master stores.
// Uneven lengths are the imbalance/divergence trade-off of P:340-342 and
// P:426 between intra-warp and inter-warp teams.
//
// Loop body: a segment starts at an arbitrary element, so each team peels a
// head of <= 3 elements up to the next 16-byte boundary, streams the aligned
// body in 128-bit units, and finishes a tail of <= 3 elements.
#include "common.cuh"
#include "np_team.cuh"

namespace cudanp {

#ifndef CUDANP_RAGGED_K
#define CUDANP_RAGGED_K 4
#endif
#ifndef CUDANP_RAGGED_UNROLL
#define CUDANP_RAGGED_UNROLL 4
#endif
constexpr int kRaggedBlock = 256;
constexpr int kRaggedK = CUDANP_RAGGED_K;  // items in flight per team
constexpr int kRaggedUnroll = CUDANP_RAGGED_UNROLL;

template <class T, class Op>
__device__ __forceinline__ V4<T> op4r(V4<T> a, V4<T> b) {
  return {Op::apply(a.x, b.x), Op::apply(a.y, b.y), Op::apply(a.z, b.z), Op::apply(a.w, b.w)};
}

// Split [b, e) into head [b, hb), aligned body units [hb, hb + 4*nu), tail.
template <class T>
__device__ __forceinline__ void split_segment(const T* in, int64_t b, int64_t e, int64_t& hb,
                                              int64_t& nu) {
  const int mis = (int)(((uintptr_t)(in + b) >> 2) & 3);  // 4-byte elements past a 16-byte line
  int64_t head = (4 - mis) & 3;
  if (head > e - b) head = e - b;
  hb = b + head;
  nu = (e - hb) >> 2;
}

// Trip count of slave `s` over n units for the distribution.
template <int S, int DIST>
__device__ __forceinline__ int64_t trips_of(const Range<S, DIST>& r) {
  if (r.end <= r.begin) return 0;
  return DIST == DIST_CYCLIC ? (r.end - r.begin + S - 1) / S : r.end - r.begin;
}

// ---------------------------------------------------------------- intra-warp
template <class T, class Op, int S, int DIST>
__global__ void __launch_bounds__(kRaggedBlock)
ragged_intra_kernel(const T* __restrict__ in, const int64_t* __restrict__ off,
                    const T* __restrict__ init, T* __restrict__ out, int64_t N) {
  constexpr int TPW = 32 / S;
  constexpr int K = kRaggedK;
  const IntraTeam<S> team;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t ntiles = (N + TPW - 1) / TPW;
  const T id = Op::template identity<T>();

  for (int64_t t0 = warp * K; t0 < ntiles; t0 += nwarps * K) {
    int64_t item[K], hb[K], nu[K], e[K], rb[K], re[K], rs[K];
    T part[K];
    int64_t trips = 0;
#pragma unroll
    for (int k = 0; k < K; ++k) {
      item[k] = (t0 + k) * TPW + team.team;
      // Sequential section (master only): read the loop bounds ...
      int64_t b0 = 0, e0 = 0;
      if (team.is_master() && item[k] < N) {
        b0 = off[item[k]];
        e0 = off[item[k] + 1];
        if (e0 < b0) e0 = b0;  // a decreasing offset pair is an empty loop
      }
      // ... and broadcast them to the slaves.
      const int64_t b = team.read_from_master(b0);
      e[k] = team.read_from_master(e0);
      split_segment(in, b, e[k], hb[k], nu[k]);
      const Range<S, DIST> r(nu[k], 4 * nu[k], 4, team.slave);
      rb[k] = r.begin; re[k] = r.end; rs[k] = r.step;
      trips = max(trips, trips_of(r));
      // head elements (<= 3), dealt cyclically
      part[k] = id;
      for (int64_t i = b + team.slave; i < hb[k]; i += S) part[k] = Op::apply(part[k], in[i]);
    }
    trips = __reduce_max_sync(kFull, (unsigned)trips);  // warp-uniform trip count
    V4<T> acc[K];
#pragma unroll
    for (int k = 0; k < K; ++k) acc[k] = {id, id, id, id};
#pragma unroll kRaggedUnroll
    for (int64_t j = 0; j < trips; ++j) {
      V4<T> v[K];
#pragma unroll
      for (int k = 0; k < K; ++k) {
        const int64_t u = rb[k] + j * rs[k];
        if (u < re[k]) v[k] = ldg4(in + hb[k] + 4 * u);
        else v[k] = {id, id, id, id};
      }
#pragma unroll
      for (int k = 0; k < K; ++k) acc[k] = op4r<T, Op>(acc[k], v[k]);
    }
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const int64_t tb = hb[k] + 4 * nu[k];
      T p = Op::apply(part[k], Op::apply(Op::apply(acc[k].x, acc[k].y), Op::apply(acc[k].z, acc[k].w)));
      for (int64_t i = tb + team.slave; i < e[k]; i += S) p = Op::apply(p, in[i]);  // tail (<= 3)
      const T res = team.template reduce<Op>(p);
      if (team.is_master() && item[k] < N) out[item[k]] = init ? Op::apply(init[item[k]], res) : res;
    }
  }
}

// ---------------------------------------------------------------- inter-warp
// blockDim = (32, S): lane = item, warp = slave; bounds and partials through smem.
template <class T, class Op, int S, int DIST>
__global__ void __launch_bounds__(32 * S)
ragged_inter_kernel(const T* __restrict__ in, const int64_t* __restrict__ off,
                    const T* __restrict__ init, T* __restrict__ out, int64_t N) {
  __shared__ int64_t slot_b[32], slot_e[32];
  __shared__ T red[S][33];
  const InterTeam<S> team;
  const int64_t ngroups = (N + 31) / 32;
  const T id = Op::template identity<T>();
  for (int64_t g = blockIdx.x; g < ngroups; g += gridDim.x) {
    const int64_t item = g * 32 + team.master;
    const bool ok = item < N;
    int64_t b0 = 0, e0 = 0;
    if (team.is_master() && ok) {
      b0 = off[item];
      e0 = off[item + 1];
      if (e0 < b0) e0 = b0;
    }
    const int64_t b = team.read_from_master(b0, slot_b);
    const int64_t e = team.read_from_master(e0, slot_e);
    int64_t hb, nu;
    split_segment(in, b, e, hb, nu);
    const Range<S, DIST> r(nu, 4 * nu, 4, team.slave);
    T p = id;
    for (int64_t i = b + team.slave; i < hb; i += S) p = Op::apply(p, in[i]);
    V4<T> acc = {id, id, id, id};
    for (int64_t u = r.begin; u < r.end; u += r.step) acc = op4r<T, Op>(acc, ldg4(in + hb + 4 * u));
    p = Op::apply(p, Op::apply(Op::apply(acc.x, acc.y), Op::apply(acc.z, acc.w)));
    const int64_t tb = hb + 4 * nu;
    for (int64_t i = tb + team.slave; i < e; i += S) p = Op::apply(p, in[i]);
    if (S == 1) {
      if (ok) out[item] = init ? Op::apply(init[item], p) : p;
      continue;
    }
    red[team.slave][team.master] = p;
    __syncthreads();
    if (team.is_master() && ok) {
      T res = red[0][team.master];
#pragma unroll
      for (int s = 1; s < S; ++s) res = Op::apply(res, red[s][team.master]);
      out[item] = init ? Op::apply(init[item], res) : res;
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------- S=1 literal
template <class T, class Op>
__global__ void __launch_bounds__(256)
ragged_literal_kernel(const T* __restrict__ in, const int64_t* __restrict__ off,
                      const T* __restrict__ init, T* __restrict__ out, int64_t N) {
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (n >= N) return;
  T acc = Op::template identity<T>();
  for (int64_t i = off[n]; i < off[n + 1]; ++i) acc = Op::apply(acc, in[i]);
  out[n] = init ? Op::apply(init[n], acc) : acc;
}

// ---------------------------------------------------------------- dispatch
template <class T, class Op, int S, int DIST>
static int launch_ragged(const T* in, const int64_t* off, const T* init, T* out, int64_t N, int map,
                         cudaStream_t st) {
  if (N == 0) return CUDANP_OK;
  if (map == MAP_INTRA) {
    auto kern = ragged_intra_kernel<T, Op, S, DIST>;
    constexpr int TPW = 32 / S;
    const int64_t ntiles = (N + TPW - 1) / TPW;
    const int64_t per_cta = (kRaggedBlock / 32) * kRaggedK;
    const int64_t grid = persistent_grid(kern, kRaggedBlock, 0, (ntiles + per_cta - 1) / per_cta);
    kern<<<(unsigned)grid, kRaggedBlock, 0, st>>>(in, off, init, out, N);
  } else {
    auto kern = ragged_inter_kernel<T, Op, S, DIST>;
    const int64_t grid = persistent_grid(kern, 32 * S, 0, (N + 31) / 32);
    kern<<<(unsigned)grid, dim3(32, S), 0, st>>>(in, off, init, out, N);
  }
  return check_launch("ragged_loop_reduce launch");
}

template <class T, class Op>
static int dispatch_ragged_t(const void* in, const int64_t* off, const void* init, void* out,
                             int64_t N, int S, int dist, int map, cudaStream_t st) {
  const T* i = (const T*)in;
  const T* ini = (const T*)init;
  T* o = (T*)out;
  CUDANP_DISPATCH_S(S, {
    return dist == DIST_CYCLIC ? launch_ragged<T, Op, kS, DIST_CYCLIC>(i, off, ini, o, N, map, st)
                               : launch_ragged<T, Op, kS, DIST_BLOCK>(i, off, ini, o, N, map, st);
  });
  return CUDANP_OK;
}

int ragged_np(const void* in, const int64_t* off, const void* init, void* out, int64_t N, int dtype,
              int op, int S, int dist, int map, cudaStream_t st) {
  if (dtype == CUDANP_F32)
    return op == CUDANP_SUM ? dispatch_ragged_t<float, OpSum>(in, off, init, out, N, S, dist, map, st)
                            : dispatch_ragged_t<float, OpMax>(in, off, init, out, N, S, dist, map, st);
  return op == CUDANP_SUM ? dispatch_ragged_t<int32_t, OpSum>(in, off, init, out, N, S, dist, map, st)
                          : dispatch_ragged_t<int32_t, OpMax>(in, off, init, out, N, S, dist, map, st);
}

int ragged_literal(const void* in, const int64_t* off, const void* init, void* out, int64_t N,
                   int dtype, int op, cudaStream_t st) {
  if (N == 0) return CUDANP_OK;
  const unsigned grid = (unsigned)((N + 255) / 256);
  if (dtype == CUDANP_F32) {
    if (op == CUDANP_SUM)
      ragged_literal_kernel<float, OpSum><<<grid, 256, 0, st>>>((const float*)in, off, (const float*)init, (float*)out, N);
    else
      ragged_literal_kernel<float, OpMax><<<grid, 256, 0, st>>>((const float*)in, off, (const float*)init, (float*)out, N);
  } else {
    if (op == CUDANP_SUM)
      ragged_literal_kernel<int32_t, OpSum><<<grid, 256, 0, st>>>((const int32_t*)in, off, (const int32_t*)init, (int32_t*)out, N);
    else
      ragged_literal_kernel<int32_t, OpMax><<<grid, 256, 0, st>>>((const int32_t*)in, off, (const int32_t*)init, (int32_t*)out, N);
  }
  return check_launch("ragged_loop_reduce literal launch");
}

}  // namespace cudanp
