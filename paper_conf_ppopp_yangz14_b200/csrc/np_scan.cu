// np_scan.cu -- batched inclusive scan: out[n*L+k] = init[n] + sum_{i<=k} in[n*L+i].
//
// The scan clause of a CUDA-NP parallel loop ("a similar approach to
// Nvidia CUDA SDK"; LIB's loop is a scan, Table 1).  The item's
// carry-in init[n] is a live-in: the master loads it and broadcasts it with
// read_from_master.  The output is in global memory, so every
// team member stores its own elements.
//
//  cyclic: in rounds of S units; each lane scans its unit locally,
//     the team runs a shfl-up Hillis-Steele scan of the unit totals, adds the
//     running carry, stores, and the carry advances by the round total (held
//     by the team's last lane).
//  block (R5): pass 1 sums each slave's contiguous chunk; an exclusive team
//     scan turns the chunk sums into offsets; pass 2 re-reads the chunk (now
//     in L1/L2) and writes the running values.  This is the register-chunk
//     partition of Fig 6c without holding the chunk in registers.
//  inter-warp: the same two schemes with shared memory instead of shfl.
#include "common.cuh"
#include "np_team.cuh"

namespace cudanp {

constexpr int kScanBlock = 256;
#ifndef CUDANP_SCAN_K
#define CUDANP_SCAN_K 2
#endif
constexpr int kScanK = CUDANP_SCAN_K;  // warp tiles per warp step (intra)

template <class T>
__device__ __forceinline__ void local_scan4(V4<T>& v) {
  v.y = OpSum::apply(v.x, v.y);
  v.z = OpSum::apply(v.y, v.z);
  v.w = OpSum::apply(v.z, v.w);
}
template <class T>
__device__ __forceinline__ V4<T> add4(V4<T> v, T a) {
  return {OpSum::apply(v.x, a), OpSum::apply(v.y, a), OpSum::apply(v.z, a), OpSum::apply(v.w, a)};
}
template <class T>
__device__ __forceinline__ T sum4(V4<T> v) {
  return OpSum::apply(OpSum::apply(v.x, v.y), OpSum::apply(v.z, v.w));
}

// ---------------------------------------------------------------- intra-warp
template <class T, int S, int DIST, bool VEC, int KT = kScanK>
__global__ void __launch_bounds__(kScanBlock)
scan_intra_kernel(const T* __restrict__ in, const T* __restrict__ init, T* __restrict__ out,
                  int64_t N, int64_t L) {
  pdl_entry();
  constexpr int TPW = 32 / S;
  constexpr int K = KT;
  constexpr int V = VEC ? 4 : 1;
  const IntraTeam<S> team;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t nunits = VEC ? (L >> 2) : L;
  const int64_t ntiles = (N + TPW - 1) / TPW;

  for (int64_t t0 = warp * K; t0 < ntiles; t0 += nwarps * K) {
    int64_t item[K];
    T carry[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      item[k] = (t0 + k) * TPW + team.team;
      // Sequential section: only the master touches the live-in,
      // then read_from_master hands it to the slaves.
      T c = T(0);
      if (init && team.is_master() && item[k] < N) c = init[item[k]];
      carry[k] = init ? team.read_from_master(c) : T(0);
    }
    if constexpr (DIST == DIST_CYCLIC) {
      const int64_t nrounds = (nunits + S - 1) / S;
#pragma unroll 2
      for (int64_t rd = 0; rd < nrounds; ++rd) {
        const int64_t u = rd * S + team.slave;
        const bool uok = u < nunits;
        if constexpr (VEC) {
          V4<T> v[K];
#pragma unroll
          for (int k = 0; k < K; ++k) {
            if (uok && item[k] < N) v[k] = ldg4(in + item[k] * L + 4 * u);
            else v[k] = {T(0), T(0), T(0), T(0)};
          }
#pragma unroll
          for (int k = 0; k < K; ++k) {
            local_scan4(v[k]);
            const T incl = team.inclusive_scan(v[k].w);
            const T excl = team.exclusive_from_inclusive(incl);
            const V4<T> o = add4(v[k], OpSum::apply(carry[k], excl));
            if (uok && item[k] < N) stg4(out + item[k] * L + 4 * u, o);
            carry[k] = OpSum::apply(carry[k], team.from_last(incl));
          }
        } else {
          T v[K];
#pragma unroll
          for (int k = 0; k < K; ++k) v[k] = (uok && item[k] < N) ? ldg1(in + item[k] * L + u) : T(0);
#pragma unroll
          for (int k = 0; k < K; ++k) {
            const T incl = team.inclusive_scan(v[k]);
            const T excl = team.exclusive_from_inclusive(incl);
            if (uok && item[k] < N) out[item[k] * L + u] = OpSum::apply(OpSum::apply(carry[k], excl), v[k]);
            carry[k] = OpSum::apply(carry[k], team.from_last(incl));
          }
        }
      }
    } else {
      const Range<S, DIST> r(nunits, L, V, team.slave);
      // pass 1: chunk sums
      T csum[K];
#pragma unroll
      for (int k = 0; k < K; ++k) csum[k] = T(0);
#pragma unroll 2
      for (int64_t u = r.begin; u < r.end; ++u) {
#pragma unroll
        for (int k = 0; k < K; ++k) {
          if (item[k] < N) {
            if constexpr (VEC) csum[k] = OpSum::apply(csum[k], sum4(ldg4(in + item[k] * L + 4 * u)));
            else csum[k] = OpSum::apply(csum[k], ldg1(in + item[k] * L + u));
          }
        }
      }
      // team scan of chunk sums -> each slave's offset
      T run[K];
#pragma unroll
      for (int k = 0; k < K; ++k) {
        const T incl = team.inclusive_scan(csum[k]);
        run[k] = OpSum::apply(carry[k], team.exclusive_from_inclusive(incl));
      }
      // pass 2: rescan the chunk with the offset
#pragma unroll 2
      for (int64_t u = r.begin; u < r.end; ++u) {
#pragma unroll
        for (int k = 0; k < K; ++k) {
          if (item[k] < N) {
            if constexpr (VEC) {
              V4<T> v = ldg4(in + item[k] * L + 4 * u);
              local_scan4(v);
              stg4(out + item[k] * L + 4 * u, add4(v, run[k]));
              run[k] = OpSum::apply(run[k], v.w);
            } else {
              run[k] = OpSum::apply(run[k], ldg1(in + item[k] * L + u));
              out[item[k] * L + u] = run[k];
            }
          }
        }
      }
    }
  }
}

// ---------------------------------------------------------------- inter-warp
// blockDim = (32, S): master = lane = item, slave = warp.  Unit totals meet in
// shared memory; every thread folds the slots below its own slave id
// (exclusive offset) and all S slots (round total).  The round total is
// recomputed redundantly by every member rather than broadcast.
template <class T, int S, int DIST, bool VEC>
__global__ void __launch_bounds__(32 * S)
scan_inter_kernel(const T* __restrict__ in, const T* __restrict__ init, T* __restrict__ out,
                  int64_t N, int64_t L) {
  pdl_entry();
  __shared__ T part[S][33];
  __shared__ T slot[32];
  constexpr int V = VEC ? 4 : 1;
  const InterTeam<S> team;
  const int64_t nunits = VEC ? (L >> 2) : L;
  const int64_t ngroups = (N + 31) / 32;

  for (int64_t g = blockIdx.x; g < ngroups; g += gridDim.x) {
    const int64_t item = g * 32 + team.master;
    const bool ok = item < N;
    T carry = T(0);
    if (init) {
      T c = T(0);
      if (team.is_master() && ok) c = init[item];
      carry = team.read_from_master(c, slot);
    }
    const T* irow = in + (ok ? item : 0) * L;
    T* orow = out + (ok ? item : 0) * L;
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
        if constexpr (VEC) local_scan4(v);
        const T tot = VEC ? v.w : v.x;
        T excl = T(0), all = T(0);
        if (S > 1) {
          part[team.slave][team.master] = tot;
          __syncthreads();
#pragma unroll
          for (int s = 0; s < S; ++s) {
            const T p = part[s][team.master];
            if (s < team.slave) excl = OpSum::apply(excl, p);
            all = OpSum::apply(all, p);
          }
          __syncthreads();
        } else {
          all = tot;
        }
        const T add = OpSum::apply(carry, excl);
        if (uok) {
          if constexpr (VEC) stg4(orow + 4 * u, add4(v, add));
          else orow[u] = OpSum::apply(add, v.x);
        }
        carry = OpSum::apply(carry, all);
      }
    } else {
      const Range<S, DIST> r(nunits, L, V, team.slave);
      T csum = T(0);
      if (ok) {
        for (int64_t u = r.begin; u < r.end; ++u) {
          if constexpr (VEC) csum = OpSum::apply(csum, sum4(ldg4(irow + 4 * u)));
          else csum = OpSum::apply(csum, ldg1(irow + u));
        }
      }
      T excl = T(0);
      if (S > 1) {
        part[team.slave][team.master] = csum;
        __syncthreads();
        for (int s = 0; s < team.slave; ++s) excl = OpSum::apply(excl, part[s][team.master]);
        __syncthreads();
      }
      T run = OpSum::apply(carry, excl);
      if (ok) {
        for (int64_t u = r.begin; u < r.end; ++u) {
          if constexpr (VEC) {
            V4<T> v = ldg4(irow + 4 * u);
            local_scan4(v);
            stg4(orow + 4 * u, add4(v, run));
            run = OpSum::apply(run, v.w);
          } else {
            run = OpSum::apply(run, ldg1(irow + u));
            orow[u] = run;
          }
        }
      }
    }
  }
}

// ---------------------------------------------------------------- S=1 literal
template <class T>
__global__ void __launch_bounds__(256)
scan_literal_kernel(const T* __restrict__ in, const T* __restrict__ init, T* __restrict__ out,
                    int64_t N, int64_t L) {
  const int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (n >= N) return;
  T acc = init ? init[n] : T(0);
  for (int64_t i = 0; i < L; ++i) {
    acc = OpSum::apply(acc, in[n * L + i]);
    out[n * L + i] = acc;
  }
}

// ---------------------------------------------------------------- dispatch
template <class T, int S, int DIST, bool VEC>
static int launch_scan_map(const T* in, const T* init, T* out, int64_t N, int64_t L, int map,
                           cudaStream_t st, LaunchInfo* info) {
  if (map == MAP_INTRA) {
   if constexpr (!kPow2<S>) {
    set_error("intra-warp teams need S = 2^k <= 32 (P:342); S = %d is built for the inter-warp map", S);
    return CUDANP_ERR_UNSUPPORTED;
   } else {
    constexpr int TPW = 32 / S;
    const int64_t ntiles = (N + TPW - 1) / TPW;
    const bool few = few_tiles(scan_intra_kernel<T, S, DIST, VEC>, kScanBlock, ntiles, kScanK);
    auto kern = few ? scan_intra_kernel<T, S, DIST, VEC, 1> : scan_intra_kernel<T, S, DIST, VEC, kScanK>;
    const int64_t per_cta = (kScanBlock / 32) * (few ? 1 : kScanK);
    const int64_t grid = persistent_grid(kern, kScanBlock, 0, (ntiles + per_cta - 1) / per_cta);
    if (info) {
      info->block_threads = kScanBlock; info->grid = grid; info->map = MAP_INTRA;
      kernel_attrs(kern, &info->regs, &info->smem);
      return CUDANP_OK;
    }
    if (N == 0 || L == 0) return CUDANP_OK;
    launch_pdl(kern, dim3((unsigned)grid), dim3(kScanBlock), 0, st, in, init, out, N, L);
   }
  } else {
    auto kern = scan_inter_kernel<T, S, DIST, VEC>;
    const int64_t grid = persistent_grid(kern, 32 * S, 0, (N + 31) / 32);
    if (info) {
      info->block_threads = 32 * S; info->grid = grid; info->map = MAP_INTER;
      kernel_attrs(kern, &info->regs, &info->smem);
      return CUDANP_OK;
    }
    if (N == 0 || L == 0) return CUDANP_OK;
    launch_pdl(kern, dim3((unsigned)grid), dim3(32, S), 0, st, in, init, out, N, L);
  }
  return check_launch("batched_loop_scan launch");
}

template <class T>
static int dispatch_scan_t(const void* in, const void* init, void* out, int64_t N, int64_t L, int S,
                           int dist, int map, bool vec, cudaStream_t st, LaunchInfo* info) {
  const T* i = (const T*)in;
  const T* ini = (const T*)init;
  T* o = (T*)out;
#define CUDANP_SCAN_BODY                                                                        \
    if (dist == DIST_CYCLIC) {                                                                  \
      return vec ? launch_scan_map<T, kS, DIST_CYCLIC, true>(i, ini, o, N, L, map, st, info)    \
                 : launch_scan_map<T, kS, DIST_CYCLIC, false>(i, ini, o, N, L, map, st, info);  \
    } else {                                                                                    \
      return vec ? launch_scan_map<T, kS, DIST_BLOCK, true>(i, ini, o, N, L, map, st, info)     \
                 : launch_scan_map<T, kS, DIST_BLOCK, false>(i, ini, o, N, L, map, st, info);   \
    }
  if (valid_inter_S(S)) {
    CUDANP_DISPATCH_S_INTER(S, { CUDANP_SCAN_BODY });
  } else {
    CUDANP_DISPATCH_S(S, { CUDANP_SCAN_BODY });
  }
#undef CUDANP_SCAN_BODY
  return CUDANP_OK;
}

int scan_cluster(const void*, const void*, void*, int64_t, int64_t, int, int, int, bool, cudaStream_t,
                 LaunchInfo*);
int scan_multi(const void*, const void*, void*, int64_t, int64_t, int, int, int, bool, cudaStream_t,
               LaunchInfo*);

int scan_np(const void* in, const void* init, void* out, int64_t N, int64_t L, int dtype, int S,
            int dist, int map, bool vec, cudaStream_t st, LaunchInfo* info) {
  if (S > 32) {
    if (map == MAP_INTER) {
      set_error("a team of S > 32 is S/32 consecutive warps: intra-warp (consecutive) map only");
      return CUDANP_ERR_UNSUPPORTED;
    }
    if (S > 1024) return scan_cluster(in, init, out, N, L, dtype, S, dist, vec, st, info);
    return scan_multi(in, init, out, N, L, dtype, S, dist, vec, st, info);
  }
  if (dtype == CUDANP_F32) return dispatch_scan_t<float>(in, init, out, N, L, S, dist, map, vec, st, info);
  return dispatch_scan_t<int32_t>(in, init, out, N, L, S, dist, map, vec, st, info);
}

int scan_literal(const void* in, const void* init, void* out, int64_t N, int64_t L, int dtype,
                 cudaStream_t st) {
  if (N == 0 || L == 0) return CUDANP_OK;
  const unsigned grid = (unsigned)((N + 255) / 256);
  if (dtype == CUDANP_F32)
    scan_literal_kernel<float><<<grid, 256, 0, st>>>((const float*)in, (const float*)init, (float*)out, N, L);
  else
    scan_literal_kernel<int32_t><<<grid, 256, 0, st>>>((const int32_t*)in, (const int32_t*)init, (int32_t*)out, N, L);
  return check_launch("batched_loop_scan literal launch");
}

}  // namespace cudanp
