// np_multi.cu -- teams larger than a warp: S in {64, 128, 256, 512, 1024}.
//
// The north star asks for "warp-shuffle reduction and scan trees with a
// shared-memory fallback when S exceeds 32".  A team of S > 32 threads is S/32
// consecutive warps of one CTA (the paper's TB enlargement up to 1024
// threads, taken to a single master per CTA when S = 1024): the
// distribution of the loop is the same (cyclic P:166 / block R5); the
// reduction and scan run as shfl trees inside each warp (intra-warp)
// and combine the S/32 warp results through shared memory (P:209,
// inter-warp).  Few outer items with long loops (MV with few rows, a batched
// reduce over few long items) get the whole GPU this way.
#include "common.cuh"
#include "np_team.cuh"

namespace cudanp {

#ifndef CUDANP_MULTI_U
#define CUDANP_MULTI_U 4
#endif
constexpr int kMultiU = CUDANP_MULTI_U;  // units per thread batched before the fold (reduce, MV)

template <class T, class Op>
__device__ __forceinline__ V4<T> mop4(V4<T> a, V4<T> b) {
  return {Op::apply(a.x, b.x), Op::apply(a.y, b.y), Op::apply(a.z, b.z), Op::apply(a.w, b.w)};
}

// ---------------------------------------------------------------- batched reduce
template <class T, class Op, int S, int DIST, bool VEC>
__global__ void __launch_bounds__(MultiShape<S>::CTA, MultiShape<S>::MINB)
reduce_multi_kernel(const T* __restrict__ in, const T* __restrict__ init, T* __restrict__ out,
                    int64_t N, int64_t L) {
  pdl_entry();
  using Sh = MultiShape<S>;
  __shared__ T sm[Sh::TEAMS * MultiTeam<S>::W];
  const MultiTeam<S> team;
  const int64_t nunits = VEC ? (L >> 2) : L;
  const Range<S, DIST> r(nunits, L, VEC ? 4 : 1, team.slave);
  const int64_t ngroups = (N + Sh::TEAMS - 1) / Sh::TEAMS;
  const T id = Op::template identity<T>();
  for (int64_t g = blockIdx.x; g < ngroups; g += gridDim.x) {
    const int64_t item = g * Sh::TEAMS + team.team;
    const bool ok = item < N;
    const T* row = in + (ok ? item : 0) * L;
    V4<T> acc = {id, id, id, id};
    if (ok) {
      int64_t u = r.begin;
      constexpr int U = kMultiU;
      for (; u + (U - 1) * r.step < r.end; u += U * r.step) {
        V4<T> v[U];
#pragma unroll
        for (int j = 0; j < U; ++j) {
          if constexpr (VEC) v[j] = ldg4(row + 4 * (u + j * r.step));
          else v[j] = {ldg1(row + u + j * r.step), id, id, id};
        }
#pragma unroll
        for (int j = 0; j < U; ++j) acc = mop4<T, Op>(acc, v[j]);
      }
      for (; u < r.end; u += r.step) {
        if constexpr (VEC) acc = mop4<T, Op>(acc, ldg4(row + 4 * u));
        else acc.x = Op::apply(acc.x, ldg1(row + u));
      }
    }
    const T p = Op::apply(Op::apply(acc.x, acc.y), Op::apply(acc.z, acc.w));
    const T res = team.template reduce<Op>(p, sm);
    if (team.is_master() && ok) out[item] = init ? Op::apply(init[item], res) : res;
  }
}

// ---------------------------------------------------------------- MV
template <int S, int DIST, bool VEC>
__global__ void __launch_bounds__(MultiShape<S>::CTA, MultiShape<S>::MINB)
mv_multi_kernel(const float* __restrict__ A, int64_t lda, const float* __restrict__ x,
                float* __restrict__ y, int64_t h, int64_t w) {
  pdl_entry();
  using Sh = MultiShape<S>;
  __shared__ float sm[Sh::TEAMS * MultiTeam<S>::W];
  const MultiTeam<S> team;
  const int64_t nunits = VEC ? (w >> 2) : w;
  const Range<S, DIST> r(nunits, w, VEC ? 4 : 1, team.slave);
  const int64_t ngroups = (h + Sh::TEAMS - 1) / Sh::TEAMS;
  for (int64_t g = blockIdx.x; g < ngroups; g += gridDim.x) {
    const int64_t rowi = g * Sh::TEAMS + team.team;
    const bool ok = rowi < h;
    const float* a = A + (ok ? rowi : 0) * lda;
    V4<float> acc = {0.f, 0.f, 0.f, 0.f};
    if (ok) {
      int64_t u = r.begin;
      constexpr int U = kMultiU;
      for (; u + (U - 1) * r.step < r.end; u += U * r.step) {
        V4<float> av[U], xv[U];
#pragma unroll
        for (int j = 0; j < U; ++j) {
          const int64_t uu = u + j * r.step;
          if constexpr (VEC) { av[j] = ldg4_stream(a + 4 * uu); xv[j] = ldg4(x + 4 * uu); }
          else { av[j].x = ldg1(a + uu); xv[j].x = ldg1(x + uu); }
        }
#pragma unroll
        for (int j = 0; j < U; ++j) {
          acc.x = fmaf(av[j].x, xv[j].x, acc.x);
          if constexpr (VEC) {
            acc.y = fmaf(av[j].y, xv[j].y, acc.y);
            acc.z = fmaf(av[j].z, xv[j].z, acc.z);
            acc.w = fmaf(av[j].w, xv[j].w, acc.w);
          }
        }
      }
      for (; u < r.end; u += r.step) {
        if constexpr (VEC) {
          const V4<float> av = ldg4_stream(a + 4 * u), xv = ldg4(x + 4 * u);
          acc.x = fmaf(av.x, xv.x, acc.x); acc.y = fmaf(av.y, xv.y, acc.y);
          acc.z = fmaf(av.z, xv.z, acc.z); acc.w = fmaf(av.w, xv.w, acc.w);
        } else {
          acc.x = fmaf(ldg1(a + u), ldg1(x + u), acc.x);
        }
      }
    }
    const float p = (acc.x + acc.y) + (acc.z + acc.w);
    const float res = team.template reduce<OpSum>(p, sm);
    if (team.is_master() && ok) y[rowi] = res;
  }
}

// ---------------------------------------------------------------- batched scan
template <class T, int S, int DIST, bool VEC>
__global__ void __launch_bounds__(MultiShape<S>::CTA, MultiShape<S>::MINB)
scan_multi_kernel(const T* __restrict__ in, const T* __restrict__ init, T* __restrict__ out,
                  int64_t N, int64_t L) {
  pdl_entry();
  using Sh = MultiShape<S>;
  __shared__ T sm[Sh::TEAMS * MultiTeam<S>::W];
  __shared__ T slot[Sh::TEAMS];
  const MultiTeam<S> team;
  constexpr int V = VEC ? 4 : 1;
  const int64_t nunits = VEC ? (L >> 2) : L;
  const int64_t ngroups = (N + Sh::TEAMS - 1) / Sh::TEAMS;
  for (int64_t g = blockIdx.x; g < ngroups; g += gridDim.x) {
    const int64_t item = g * Sh::TEAMS + team.team;
    const bool ok = item < N;
    const T* irow = in + (ok ? item : 0) * L;
    T* orow = out + (ok ? item : 0) * L;
    T carry = T(0);
    if (init) {  // live-in: the master loads it and broadcasts it
      T c = T(0);
      if (team.is_master() && ok) c = init[item];
      carry = team.read_from_master(c, slot);
    }
    if constexpr (DIST == DIST_CYCLIC) {
      const int64_t nrounds = (nunits + S - 1) / S;
      for (int64_t rd = 0; rd < nrounds; ++rd) {
        const int64_t u = rd * S + team.slave;
        const bool uok = ok && u < nunits;
        V4<T> v = {T(0), T(0), T(0), T(0)};
        if (uok) {
          if constexpr (VEC) v = ldg4(irow + 4 * u);
          else v.x = ldg1(irow + u);
        }
        if constexpr (VEC) {
          v.y = OpSum::apply(v.x, v.y); v.z = OpSum::apply(v.y, v.z); v.w = OpSum::apply(v.z, v.w);
        }
        const T tot = VEC ? v.w : v.x;
        T all;
        const T add = OpSum::apply(carry, team.exclusive_scan(tot, sm, &all));  // carry + exclusive prefix
        if (uok) {
          if constexpr (VEC)
            stg4(orow + 4 * u, V4<T>{OpSum::apply(v.x, add), OpSum::apply(v.y, add),
                                     OpSum::apply(v.z, add), OpSum::apply(v.w, add)});
          else orow[u] = OpSum::apply(add, v.x);
        }
        carry = OpSum::apply(carry, all);
      }
    } else {
      const Range<S, DIST> r(nunits, L, V, team.slave);
      T csum = T(0);
      if (ok) {
        for (int64_t u = r.begin; u < r.end; ++u) {
          if constexpr (VEC) {
            const V4<T> v = ldg4(irow + 4 * u);
            csum = OpSum::apply(csum, OpSum::apply(OpSum::apply(v.x, v.y), OpSum::apply(v.z, v.w)));
          } else {
            csum = OpSum::apply(csum, ldg1(irow + u));
          }
        }
      }
      T all;
      T run = OpSum::apply(carry, team.exclusive_scan(csum, sm, &all));
      if (ok) {
        for (int64_t u = r.begin; u < r.end; ++u) {
          if constexpr (VEC) {
            V4<T> v = ldg4(irow + 4 * u);
            v.x = OpSum::apply(run, v.x); v.y = OpSum::apply(v.x, v.y);
            v.z = OpSum::apply(v.y, v.z); v.w = OpSum::apply(v.z, v.w);
            stg4(orow + 4 * u, v);
            run = v.w;
          } else {
            run = OpSum::apply(run, ldg1(irow + u));
            orow[u] = run;
          }
        }
      }
    }
  }
}

// ---------------------------------------------------------------- dispatch
#define CUDANP_DISPATCH_BIG_S(S, ...)                        \
  switch (S) {                                               \
    case 64: { constexpr int kS = 64; __VA_ARGS__; } break;     \
    case 128: { constexpr int kS = 128; __VA_ARGS__; } break;   \
    case 256: { constexpr int kS = 256; __VA_ARGS__; } break;   \
    case 512: { constexpr int kS = 512; __VA_ARGS__; } break;   \
    case 1024: { constexpr int kS = 1024; __VA_ARGS__; } break; \
    default: return fail_invalid("S must be 64, 128, 256, 512 or 1024 for a multi-warp team"); \
  }

template <class K>
static int64_t multi_grid(K kern, int cta, int64_t groups) {
  return persistent_grid(kern, cta, 0, groups);
}

template <class T, class Op>
static int reduce_multi_t(const void* in, const void* init, void* out, int64_t N, int64_t L, int S,
                          int dist, bool vec, cudaStream_t st, LaunchInfo* info) {
  CUDANP_DISPATCH_BIG_S(S, {
    using Sh = MultiShape<kS>;
    auto kern = dist == DIST_CYCLIC
                    ? (vec ? reduce_multi_kernel<T, Op, kS, DIST_CYCLIC, true> : reduce_multi_kernel<T, Op, kS, DIST_CYCLIC, false>)
                    : (vec ? reduce_multi_kernel<T, Op, kS, DIST_BLOCK, true> : reduce_multi_kernel<T, Op, kS, DIST_BLOCK, false>);
    const int64_t grid = multi_grid(kern, Sh::CTA, (N + Sh::TEAMS - 1) / Sh::TEAMS);
    if (info) {
      info->block_threads = Sh::CTA; info->grid = grid; info->map = MAP_INTRA;
      kernel_attrs(kern, &info->regs, &info->smem);
      return CUDANP_OK;
    }
    if (N == 0) return CUDANP_OK;
    launch_pdl(kern, dim3((unsigned)grid), dim3(Sh::CTA), 0, st, (const T*)in, (const T*)init, (T*)out, N, L);
    return check_launch("batched_loop_reduce (multi-warp team) launch");
  });
  return CUDANP_OK;
}

int reduce_multi(const void* in, const void* init, void* out, int64_t N, int64_t L, int dtype,
                 int op, int S, int dist, bool vec, cudaStream_t st, LaunchInfo* info) {
  if (dtype == CUDANP_F32)
    return op == CUDANP_SUM ? reduce_multi_t<float, OpSum>(in, init, out, N, L, S, dist, vec, st, info)
                            : reduce_multi_t<float, OpMax>(in, init, out, N, L, S, dist, vec, st, info);
  return op == CUDANP_SUM ? reduce_multi_t<int32_t, OpSum>(in, init, out, N, L, S, dist, vec, st, info)
                          : reduce_multi_t<int32_t, OpMax>(in, init, out, N, L, S, dist, vec, st, info);
}

template <class T>
static int scan_multi_t(const void* in, const void* init, void* out, int64_t N, int64_t L, int S,
                        int dist, bool vec, cudaStream_t st, LaunchInfo* info) {
  CUDANP_DISPATCH_BIG_S(S, {
    using Sh = MultiShape<kS>;
    auto kern = dist == DIST_CYCLIC
                    ? (vec ? scan_multi_kernel<T, kS, DIST_CYCLIC, true> : scan_multi_kernel<T, kS, DIST_CYCLIC, false>)
                    : (vec ? scan_multi_kernel<T, kS, DIST_BLOCK, true> : scan_multi_kernel<T, kS, DIST_BLOCK, false>);
    const int64_t grid = multi_grid(kern, Sh::CTA, (N + Sh::TEAMS - 1) / Sh::TEAMS);
    if (info) {
      info->block_threads = Sh::CTA; info->grid = grid; info->map = MAP_INTRA;
      kernel_attrs(kern, &info->regs, &info->smem);
      return CUDANP_OK;
    }
    if (N == 0 || L == 0) return CUDANP_OK;
    launch_pdl(kern, dim3((unsigned)grid), dim3(Sh::CTA), 0, st, (const T*)in, (const T*)init, (T*)out, N, L);
    return check_launch("batched_loop_scan (multi-warp team) launch");
  });
  return CUDANP_OK;
}

int scan_multi(const void* in, const void* init, void* out, int64_t N, int64_t L, int dtype, int S,
               int dist, bool vec, cudaStream_t st, LaunchInfo* info) {
  return dtype == CUDANP_F32 ? scan_multi_t<float>(in, init, out, N, L, S, dist, vec, st, info)
                             : scan_multi_t<int32_t>(in, init, out, N, L, S, dist, vec, st, info);
}

int mv_multi(const float* A, int64_t lda, const float* x, float* y, int64_t h, int64_t w, int S,
             int dist, bool vec, cudaStream_t st, LaunchInfo* info) {
  CUDANP_DISPATCH_BIG_S(S, {
    using Sh = MultiShape<kS>;
    auto kern = dist == DIST_CYCLIC ? (vec ? mv_multi_kernel<kS, DIST_CYCLIC, true> : mv_multi_kernel<kS, DIST_CYCLIC, false>)
                                    : (vec ? mv_multi_kernel<kS, DIST_BLOCK, true> : mv_multi_kernel<kS, DIST_BLOCK, false>);
    const int64_t grid = multi_grid(kern, Sh::CTA, (h + Sh::TEAMS - 1) / Sh::TEAMS);
    if (info) {
      info->block_threads = Sh::CTA; info->grid = grid; info->map = MAP_INTRA;
      kernel_attrs(kern, &info->regs, &info->smem);
      return CUDANP_OK;
    }
    if (h == 0) return CUDANP_OK;
    // Launched WITHOUT programmatic dependent launch: its CTAs launched early
    // would co-reside with a preceding TMA TMV's CTAs (which leave registers
    // free on every SM) and the C2 step (TMV then MV, repeated) loses 3-4 %;
    // launched plainly they start on SMs the TMV has left (A/B,
    // tools/exp_pdl_ab.py: step 7.07 -> 7.33 TB/s; MV repeated alone -1 %).
    launch_pdl_if(false, kern, dim3((unsigned)grid), dim3(Sh::CTA), 0, st, A, lda, x, y, h, w);
    return check_launch("mv (multi-warp team) launch");
  });
  return CUDANP_OK;
}

}  // namespace cudanp
