// np_reduce.cu -- batched loop-reduce: out[n] = init[n] (op) fold_i in[n*L+i].
//
// One outer item = one original thread whose parallel loop (trip count L)
// carries a reduction clause (Fig 6d).  CUDA-NP
// gives the item a team of S threads; each runs its share of the loop
// (cyclic P:166 / block R5), the team combines the partials (shfl for
// intra-warp, shared memory for inter-warp) and the master alone
// finishes the item.
//
// B200 design: the loop body is an HBM stream, so each
// lane issues 128-bit read-only loads (LDG.E.128.CONSTANT) when rows are
// 16-byte aligned, keeps K items in flight (memory-level parallelism), and the
// grid is persistent: a whole number of waves of resident CTAs that stride
// over items.
#include "common.cuh"
#include "np_team.cuh"

#include <type_traits>

namespace cudanp {

constexpr int kReduceBlock = 256;  // intra-warp CTA: 8 warps
#ifndef CUDANP_REDUCE_K
#define CUDANP_REDUCE_K 2
#endif
constexpr int kReduceK = CUDANP_REDUCE_K;  // warp tiles in flight per warp (intra)

template <class T, class Op>
__device__ __forceinline__ T fold4(V4<T> v) {
  return Op::apply(Op::apply(v.x, v.y), Op::apply(v.z, v.w));
}
template <class T, class Op>
__device__ __forceinline__ V4<T> op4(V4<T> a, V4<T> b) {
  return {Op::apply(a.x, b.x), Op::apply(a.y, b.y), Op::apply(a.z, b.z), Op::apply(a.w, b.w)};
}

// Team-reduction backend (the Fig 16 ablation): 0 = shfl
// butterfly (default), 1 = shared memory, 2 = redux.sync.
enum { RB_SHFL = 0, RB_SMEM = 1, RB_REDUX = 2 };

template <class T, class Op>
__device__ __forceinline__ T redux_op(T v, unsigned mask) {
  if constexpr (std::is_same<Op, OpSum>::value) return Redux::sum(v, mask);
  else return Redux::max(v, mask);
}

// ---------------------------------------------------------------- intra-warp
// Team = S lanes; a warp holds TPW = 32/S teams = TPW items ("warp tile").
// Each warp processes K consecutive warp tiles per step of a grid-stride
// loop, so a lane has K independent rows in flight.
#ifndef CUDANP_REDUCE_MINB
#define CUDANP_REDUCE_MINB 1
#endif
template <class T, class Op, int S, int DIST, bool VEC, int RB = RB_SHFL, int KT = kReduceK,
          bool W8 = false>
__global__ void __launch_bounds__(kReduceBlock, CUDANP_REDUCE_MINB)
reduce_intra_kernel(const T* __restrict__ in, const T* __restrict__ init, T* __restrict__ out,
                    int64_t N, int64_t L) {
  pdl_entry();
  __shared__ T slots[RB == RB_SMEM ? kReduceBlock : 1];
  constexpr int TPW = 32 / S;
  constexpr int K = KT;
  constexpr int V = W8 ? 8 : (VEC ? 4 : 1);  // elements per unit (one load)
  const IntraTeam<S> team;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t nunits = L / V;
  // Iteration share of this slave: uniform index math, recomputed by every
  // slave instead of broadcast.
  const Range<S, DIST> r(nunits, L, V, team.slave);
  const int64_t ntiles = (N + TPW - 1) / TPW;

  for (int64_t t0 = warp * K; t0 < ntiles; t0 += nwarps * K) {
#if defined(CUDANP_L2PF)
    if constexpr (VEC) {
      // The warp's K tiles CUDANP_L2PF steps ahead are one contiguous block of
      // items: prefetch it into L2 so more bytes are in flight than the
      // registers of the resident warps hold.
      const int64_t tp = t0 + (int64_t)CUDANP_L2PF * nwarps * K;
      if (tp < ntiles && team.lane == 0) {
        const int64_t i0 = tp * TPW, i1 = (tp + K) * TPW < N ? (tp + K) * TPW : N;
        prefetch_l2(in + i0 * L, (uint32_t)((i1 - i0) * L * (int64_t)sizeof(T)));
      }
    }
#endif
    int64_t item[K];
    const T* row[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      item[k] = (t0 + k) * TPW + team.team;
      row[k] = in + (item[k] < N ? item[k] : 0) * L;
    }
    T part[K];
    if constexpr (W8) {
      // 256-bit units (rows 32-byte aligned, L % 8 == 0): 8 accumulators per lane
      V8<T> acc[K];
#pragma unroll
      for (int k = 0; k < K; ++k)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[k].v[j] = Op::template identity<T>();
#pragma unroll 2
      for (int64_t u = r.begin; u < r.end; u += r.step) {
        V8<T> v[K];
#pragma unroll
        for (int k = 0; k < K; ++k)
          if (item[k] < N) v[k] = ldg8(row[k] + 8 * u);
#pragma unroll
        for (int k = 0; k < K; ++k)
          if (item[k] < N)
#pragma unroll
            for (int j = 0; j < 8; ++j) acc[k].v[j] = Op::apply(acc[k].v[j], v[k].v[j]);
      }
#pragma unroll
      for (int k = 0; k < K; ++k) {
        const V8<T>& a = acc[k];
        part[k] = Op::apply(Op::apply(Op::apply(a.v[0], a.v[1]), Op::apply(a.v[2], a.v[3])),
                            Op::apply(Op::apply(a.v[4], a.v[5]), Op::apply(a.v[6], a.v[7])));
      }
    } else if constexpr (VEC) {
      V4<T> acc[K];
#pragma unroll
      for (int k = 0; k < K; ++k) {
        const T id = Op::template identity<T>();
        acc[k] = {id, id, id, id};
      }
      // Parallel loop section: every team member active.
#pragma unroll 2
      for (int64_t u = r.begin; u < r.end; u += r.step) {
        V4<T> v[K];
#pragma unroll
        for (int k = 0; k < K; ++k)
          if (item[k] < N) v[k] = ldg4(row[k] + 4 * u);
#pragma unroll
        for (int k = 0; k < K; ++k)
          if (item[k] < N) acc[k] = op4<T, Op>(acc[k], v[k]);
      }
#pragma unroll
      for (int k = 0; k < K; ++k) part[k] = fold4<T, Op>(acc[k]);
    } else {
#pragma unroll
      for (int k = 0; k < K; ++k) part[k] = Op::template identity<T>();
#pragma unroll 4
      for (int64_t u = r.begin; u < r.end; u += r.step) {
        T v[K];
#pragma unroll
        for (int k = 0; k < K; ++k)
          if (item[k] < N) v[k] = ldg1(row[k] + u);
#pragma unroll
        for (int k = 0; k < K; ++k)
          if (item[k] < N) part[k] = Op::apply(part[k], v[k]);
      }
    }
    // Live-out reduction over the team (shfl), then the master-only
    // epilogue: combine with init[n] and store.
#pragma unroll
    for (int k = 0; k < K; ++k) {
      T res;
      if constexpr (RB == RB_SMEM) res = team.template reduce_smem<Op>(part[k], slots + (threadIdx.x & ~31));
      else if constexpr (RB == RB_REDUX) res = redux_op<T, Op>(part[k], team.segment_mask());
      else res = team.template reduce<Op>(part[k]);
      if (team.is_master() && item[k] < N)
        out[item[k]] = init ? Op::apply(init[item[k]], res) : res;
    }
  }
}

// ---------------------------------------------------------------- inter-warp
// blockDim = (32, S): master = threadIdx.x (32 items per CTA step), slave =
// threadIdx.y.  Partials meet in shared memory; the master warp
// (slave 0) folds them in slave order and stores.
template <class T, class Op, int S, int DIST, bool VEC>
__global__ void __launch_bounds__(32 * S)
reduce_inter_kernel(const T* __restrict__ in, const T* __restrict__ init, T* __restrict__ out,
                    int64_t N, int64_t L) {
  pdl_entry();
  __shared__ T red[S][33];
  const InterTeam<S> team;
  const int64_t nunits = VEC ? (L >> 2) : L;
  const Range<S, DIST> r(nunits, L, VEC ? 4 : 1, team.slave);
  const int64_t ngroups = (N + 31) / 32;

  for (int64_t g = blockIdx.x; g < ngroups; g += gridDim.x) {
    const int64_t item = g * 32 + team.master;
    const bool ok = item < N;
    const T* row = in + (ok ? item : 0) * L;
    T part;
    if constexpr (VEC) {
      const T id = Op::template identity<T>();
      V4<T> acc = {id, id, id, id};
      if (ok) {
        // 4 loads in flight before the fold (the same batching as tmv_rows)
        int64_t u = r.begin;
        for (; u + 3 * r.step < r.end; u += 4 * r.step) {
          V4<T> v[4];
#pragma unroll
          for (int j = 0; j < 4; ++j) v[j] = ldg4(row + 4 * (u + j * r.step));
#pragma unroll
          for (int j = 0; j < 4; ++j) acc = op4<T, Op>(acc, v[j]);
        }
        for (; u < r.end; u += r.step) acc = op4<T, Op>(acc, ldg4(row + 4 * u));
      }
      part = fold4<T, Op>(acc);
    } else {
      part = Op::template identity<T>();
      if (ok) {
        int64_t u = r.begin;
        for (; u + 3 * r.step < r.end; u += 4 * r.step) {
          T v[4];
#pragma unroll
          for (int j = 0; j < 4; ++j) v[j] = ldg1(row + u + j * r.step);
#pragma unroll
          for (int j = 0; j < 4; ++j) part = Op::apply(part, v[j]);
        }
        for (; u < r.end; u += r.step) part = Op::apply(part, ldg1(row + u));
      }
    }
    if (S == 1) {
      if (ok) out[item] = init ? Op::apply(init[item], part) : part;
      continue;
    }
    red[team.slave][team.master] = part;
    __syncthreads();
    if (team.is_master()) {
      T res = red[0][team.master];
#pragma unroll
      for (int s = 1; s < S; ++s) res = Op::apply(res, red[s][team.master]);
      if (ok) out[item] = init ? Op::apply(init[item], res) : res;
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------- S=1 literal
// Fig 2's shape applied to the reduce: one thread per item, a scalar serial
// loop, no vector loads, no persistent grid (the paper's baseline kernel).
template <class T, class Op>
__global__ void __launch_bounds__(256)
reduce_literal_kernel(const T* __restrict__ in, const T* __restrict__ init, T* __restrict__ out,
                      int64_t N, int64_t L) {
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (n >= N) return;
  T acc = Op::template identity<T>();
  for (int64_t i = 0; i < L; ++i) acc = Op::apply(acc, in[n * L + i]);
  out[n] = init ? Op::apply(init[n], acc) : acc;
}

// ---------------------------------------------------------------- dispatch
template <class T, class Op, int S, int DIST, bool VEC>
static int launch_reduce_map(const T* in, const T* init, T* out, int64_t N, int64_t L, int map,
                             cudaStream_t st, LaunchInfo* info) {
  if (map == MAP_INTRA) {
   if constexpr (!kPow2<S>) {
    set_error("intra-warp teams need S = 2^k <= 32 (P:342); S = %d is built for the inter-warp map", S);
    return CUDANP_ERR_UNSUPPORTED;
   } else {
    constexpr int TPW = 32 / S;
    const int64_t ntiles = (N + TPW - 1) / TPW;
    const bool few = few_tiles(reduce_intra_kernel<T, Op, S, DIST, VEC>, kReduceBlock, ntiles, kReduceK);
    auto kern = few ? reduce_intra_kernel<T, Op, S, DIST, VEC, RB_SHFL, 1>
                    : reduce_intra_kernel<T, Op, S, DIST, VEC, RB_SHFL, kReduceK>;
#if defined(CUDANP_LDG256)
    if constexpr (VEC) {  // 256-bit units when rows are 32-byte aligned
      if (L % 8 == 0 && ((uintptr_t)in & 31) == 0)
        kern = few ? reduce_intra_kernel<T, Op, S, DIST, true, RB_SHFL, 1, true>
                   : reduce_intra_kernel<T, Op, S, DIST, true, RB_SHFL, kReduceK, true>;
    }
#endif
    const int64_t per_cta = (kReduceBlock / 32) * (few ? 1 : kReduceK);
    const int64_t grid = persistent_grid(kern, kReduceBlock, 0, (ntiles + per_cta - 1) / per_cta);
    if (info) {
      info->block_threads = kReduceBlock; info->grid = grid; info->map = MAP_INTRA;
      kernel_attrs(kern, &info->regs, &info->smem);
      return CUDANP_OK;
    }
    if (N == 0) return CUDANP_OK;
    launch_pdl(kern, dim3((unsigned)grid), dim3(kReduceBlock), 0, st, in, init, out, N, L);
   }
  } else {
    auto kern = reduce_inter_kernel<T, Op, S, DIST, VEC>;
    const int64_t grid = persistent_grid(kern, 32 * S, 0, (N + 31) / 32);
    if (info) {
      info->block_threads = 32 * S; info->grid = grid; info->map = MAP_INTER;
      kernel_attrs(kern, &info->regs, &info->smem);
      return CUDANP_OK;
    }
    if (N == 0) return CUDANP_OK;
    launch_pdl(kern, dim3((unsigned)grid), dim3(32, S), 0, st, in, init, out, N, L);
  }
  return check_launch("batched_loop_reduce launch");
}

template <class T, class Op>
static int dispatch_reduce_t(const void* in, const void* init, void* out, int64_t N, int64_t L,
                             int S, int dist, int map, bool vec, cudaStream_t st, LaunchInfo* info) {
  const T* i = (const T*)in;
  const T* ini = (const T*)init;
  T* o = (T*)out;
#define CUDANP_REDUCE_BODY                                                                          \
    if (dist == DIST_CYCLIC) {                                                                      \
      return vec ? launch_reduce_map<T, Op, kS, DIST_CYCLIC, true>(i, ini, o, N, L, map, st, info)  \
                 : launch_reduce_map<T, Op, kS, DIST_CYCLIC, false>(i, ini, o, N, L, map, st, info); \
    } else {                                                                                        \
      return vec ? launch_reduce_map<T, Op, kS, DIST_BLOCK, true>(i, ini, o, N, L, map, st, info)   \
                 : launch_reduce_map<T, Op, kS, DIST_BLOCK, false>(i, ini, o, N, L, map, st, info);  \
    }
  if (valid_inter_S(S)) {
    CUDANP_DISPATCH_S_INTER(S, { CUDANP_REDUCE_BODY });
  } else {
    CUDANP_DISPATCH_S(S, { CUDANP_REDUCE_BODY });
  }
#undef CUDANP_REDUCE_BODY
  return CUDANP_OK;
}

int reduce_multi(const void*, const void*, void*, int64_t, int64_t, int, int, int, int, bool,
                 cudaStream_t, LaunchInfo*);

int reduce_uniform_peel(const void*, const void*, void*, int64_t, int64_t, int, int, int, int,
                        cudaStream_t, LaunchInfo*);
int reduce_cluster(const void*, const void*, void*, int64_t, int64_t, int, int, int, int, bool,
                   cudaStream_t, LaunchInfo*);

int reduce_np(const void* in, const void* init, void* out, int64_t N, int64_t L, int dtype, int op,
              int S, int dist, int map, bool vec, cudaStream_t st, LaunchInfo* info) {
  // Rows that are not 16-byte aligned (L % 4 != 0, e.g. Table 1's L = 150):
  // intra-warp teams peel each row to its 16-byte boundary and stream the
  // body in 128-bit units (np_ragged.cu, UNI form) instead of scalar loads.
  if (!vec && S <= 32 && map == MAP_INTRA && L > 0 && ((uintptr_t)in & 3) == 0)
    return reduce_uniform_peel(in, init, out, N, L, dtype, op, S, dist, st, info);
  if (S > 32) {
    if (map == MAP_INTER) {
      set_error("a team of S > 32 is S/32 consecutive warps: intra-warp (consecutive) map only");
      return CUDANP_ERR_UNSUPPORTED;
    }
    if (S > 1024) return reduce_cluster(in, init, out, N, L, dtype, op, S, dist, vec, st, info);
    return reduce_multi(in, init, out, N, L, dtype, op, S, dist, vec, st, info);
  }
  if (dtype == CUDANP_F32)
    return op == CUDANP_SUM
               ? dispatch_reduce_t<float, OpSum>(in, init, out, N, L, S, dist, map, vec, st, info)
               : dispatch_reduce_t<float, OpMax>(in, init, out, N, L, S, dist, map, vec, st, info);
  return op == CUDANP_SUM
             ? dispatch_reduce_t<int32_t, OpSum>(in, init, out, N, L, S, dist, map, vec, st, info)
             : dispatch_reduce_t<int32_t, OpMax>(in, init, out, N, L, S, dist, map, vec, st, info);
}

// Fig 16 ablation entry: intra-warp, cyclic, 128-bit path, chosen backend.
template <class T, class Op, int RB>
static int launch_reduce_backend(const void* in, const void* init, void* out, int64_t N, int64_t L,
                                 int S, cudaStream_t st) {
  CUDANP_DISPATCH_S(S, {
    auto kern = reduce_intra_kernel<T, Op, kS, DIST_CYCLIC, true, RB>;
    constexpr int TPW = 32 / kS;
    const int64_t ntiles = (N + TPW - 1) / TPW;
    const int64_t per_cta = (kReduceBlock / 32) * kReduceK;
    const int64_t grid = persistent_grid(kern, kReduceBlock, 0, (ntiles + per_cta - 1) / per_cta);
    if (N == 0) return CUDANP_OK;
    launch_pdl(kern, dim3((unsigned)grid), dim3(kReduceBlock), 0, st, (const T*)in, (const T*)init, (T*)out, N, L);
    return check_launch("batched_loop_reduce_backend launch");
  });
  return CUDANP_OK;
}

template <class T, class Op>
static int reduce_backend_t(const void* in, const void* init, void* out, int64_t N, int64_t L, int S,
                            int backend, cudaStream_t st) {
  if (backend == RB_SHFL) return launch_reduce_backend<T, Op, RB_SHFL>(in, init, out, N, L, S, st);
  if (backend == RB_SMEM) return launch_reduce_backend<T, Op, RB_SMEM>(in, init, out, N, L, S, st);
  if constexpr (std::is_same<T, float>::value && std::is_same<Op, OpSum>::value) {
    set_error("redux.sync has no fp32 add (fp32 min/max and int32 add/max only)");
    return CUDANP_ERR_UNSUPPORTED;
  } else {
    return launch_reduce_backend<T, Op, RB_REDUX>(in, init, out, N, L, S, st);
  }
}

int reduce_backend(const void* in, const void* init, void* out, int64_t N, int64_t L, int dtype,
                   int op, int S, int backend, cudaStream_t st) {
  if (dtype == CUDANP_F32)
    return op == CUDANP_SUM ? reduce_backend_t<float, OpSum>(in, init, out, N, L, S, backend, st)
                            : reduce_backend_t<float, OpMax>(in, init, out, N, L, S, backend, st);
  return op == CUDANP_SUM ? reduce_backend_t<int32_t, OpSum>(in, init, out, N, L, S, backend, st)
                          : reduce_backend_t<int32_t, OpMax>(in, init, out, N, L, S, backend, st);
}

int reduce_literal(const void* in, const void* init, void* out, int64_t N, int64_t L, int dtype,
                   int op, cudaStream_t st) {
  if (N == 0) return CUDANP_OK;
  const unsigned grid = (unsigned)((N + 255) / 256);
  if (dtype == CUDANP_F32) {
    if (op == CUDANP_SUM)
      reduce_literal_kernel<float, OpSum><<<grid, 256, 0, st>>>((const float*)in, (const float*)init, (float*)out, N, L);
    else
      reduce_literal_kernel<float, OpMax><<<grid, 256, 0, st>>>((const float*)in, (const float*)init, (float*)out, N, L);
  } else {
    if (op == CUDANP_SUM)
      reduce_literal_kernel<int32_t, OpSum><<<grid, 256, 0, st>>>((const int32_t*)in, (const int32_t*)init, (int32_t*)out, N, L);
    else
      reduce_literal_kernel<int32_t, OpMax><<<grid, 256, 0, st>>>((const int32_t*)in, (const int32_t*)init, (int32_t*)out, N, L);
  }
  return check_launch("batched_loop_reduce literal launch");
}

}  // namespace cudanp
