// np_cluster.cu -- teams larger than a CTA: S in {2048, 4096, 8192}, one team
// per thread-block cluster of 8 CTAs (S/8 threads each).
//
// The paper enlarges a thread block "up to 1024" threads to hold the slaves
// and combines inter-warp live-outs through shared memory (P:203,
// P:209).  On sm_100a a thread-block cluster gives a group of CTAs on one GPC
// distributed shared memory and a hardware barrier, so the same construction
// extends one level up: a master's team is the cluster.  The loop is dealt
// over all S = 8 x CTA threads exactly as for every other team (cyclic P:166 /
// block R5, slave id = cluster rank x CTA + thread), each CTA folds its
// threads' partials with shfl + shared memory (the multi-warp team), each
// CTA's partial is stored into the master CTA's shared memory over DSMEM,
// and after one cluster barrier the master (rank 0, thread 0) folds the eight
// partials in rank order and stores the item.
//
// This is for the case the paper motivates NP with: few outer items with long
// loops, where even a 1024-thread team per item leaves SMs idle or unevenly
// loaded (e.g. 256 items on 148 SMs).  With a cluster per item the hardware
// block scheduler balances 8x more, smaller CTAs.
#include <cooperative_groups.h>

#include "common.cuh"
#include "np_team.cuh"

namespace cg = cooperative_groups;

namespace cudanp {

constexpr int kClusterCtas = 8;  // portable cluster size

template <class T>
__device__ __forceinline__ T sum4(V4<T> v) {
  return OpSum::apply(OpSum::apply(v.x, v.y), OpSum::apply(v.z, v.w));
}
// Exclusive prefix inside a warp from the inclusive one: the previous lane's
// inclusive value (0 for lane 0).  Taken by a shuffle, not as incl - own, so
// an fp32 exclusive value is the sum of the earlier lanes' terms themselves
// (no cancellation error).  Every lane of the warp must call it.
template <class T>
__device__ __forceinline__ T warp_prev(T incl) {
  const T t = __shfl_up_sync(kFull, incl, 1);
  return (threadIdx.x & 31) == 0 ? T(0) : t;
}

template <class T, class Op>
__device__ __forceinline__ V4<T> cop4(V4<T> a, V4<T> b) {
  return {Op::apply(a.x, b.x), Op::apply(a.y, b.y), Op::apply(a.z, b.z), Op::apply(a.w, b.w)};
}

// The cluster-wide team reduction of one item.  Every thread of the cluster
// calls it with its partial p; the master (rank 0, thread 0) gets the team's
// result in *res and true.  Level 1: shfl inside each warp; level 2:
// the CTA's warps through shared memory; level 3: each CTA's partial
// is stored into the master CTA's slot over DSMEM, one cluster barrier, and
// the master folds the eight partials in rank order.  Slots are
// double-buffered by item parity: slots [par] are rewritten two items later,
// after the next cluster barrier, which rank 0 reaches only after reading
// them.  wsum is double-buffered the same way, so a warp's write for item
// i+1 never meets the master thread's read for item i even under CTA-barrier
// reasoning alone (racecheck does not model the cluster barrier).  The first call waits on the arrive issued at kernel entry (a CTA may
// touch another CTA's shared memory only once that CTA is known to run).
template <class Op, int W, class T>
__device__ __forceinline__ bool cluster_team_reduce(T p, T* wsum, T (*part)[kClusterCtas], T* master_part,
                                                    int par, int rank, bool& started, T* res) {
  cg::cluster_group cluster = cg::this_cluster();
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) p = Op::apply(p, __shfl_xor_sync(kFull, p, o));
  wsum += par * W;
  if (lane == 0) wsum[wid] = p;
  if (!started) {  // CTA-uniform
    asm volatile("barrier.cluster.wait.aligned;" ::: "memory");
    started = true;
  }
  __syncthreads();
  if (tid == 0) {
    T c = wsum[0];
#pragma unroll
    for (int k = 1; k < W; ++k) c = Op::apply(c, wsum[k]);
    master_part[par * kClusterCtas + rank] = c;
  }
  cluster.sync();  // release/acquire: every slot is visible to rank 0; wsum reusable
  if (rank == 0 && tid == 0) {
    T r = part[par][0];
#pragma unroll
    for (int k = 1; k < kClusterCtas; ++k) r = Op::apply(r, part[par][k]);
    *res = r;
    return true;
  }
  return false;
}

__device__ __forceinline__ void cluster_arrive_relaxed() {
  asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
}
__device__ __forceinline__ void cluster_wait() {
  asm volatile("barrier.cluster.wait.aligned;" ::: "memory");
}

// ---------------------------------------------------------------- batched reduce
template <class T, class Op, int S, int DIST, bool VEC>
__global__ void __launch_bounds__(S / kClusterCtas, 4096 / S > 0 ? 4096 / S : 1)  // <= 128 registers
reduce_cluster_kernel(const T* __restrict__ in, const T* __restrict__ init, T* __restrict__ out,
                      int64_t N, int64_t L) {
  pdl_entry();
  constexpr int CTA = S / kClusterCtas;
  __shared__ T wsum[2 * (CTA / 32)];
  __shared__ T part[2][kClusterCtas];  // the master CTA's receive slots
  cg::cluster_group cluster = cg::this_cluster();
  const int rank = (int)cluster.block_rank();
  const int slave = rank * CTA + threadIdx.x;  // slave id within the cluster-wide team
  const int64_t nunits = VEC ? (L >> 2) : L;
  const Range<S, DIST> r(nunits, L, VEC ? 4 : 1, slave);
  const int64_t cid = blockIdx.x / kClusterCtas, ncl = gridDim.x / kClusterCtas;
  const T id = Op::template identity<T>();
  T* master_part = cluster.map_shared_rank(&part[0][0], 0);
  cluster_arrive_relaxed();  // waited for before the first DSMEM store
  bool started = false;
  int par = 0;
  for (int64_t item = cid; item < N; item += ncl, par ^= 1) {
    const T* row = in + item * L;
    V4<T> acc = {id, id, id, id};
    int64_t u = r.begin;
    constexpr int U = 8;  // 128 B in flight per thread: few CTAs per SM carry the stream
    for (; u + (U - 1) * r.step < r.end; u += U * r.step) {
      V4<T> v[U];
#pragma unroll
      for (int j = 0; j < U; ++j) {
        if constexpr (VEC) v[j] = ldg4(row + 4 * (u + j * r.step));
        else v[j] = {ldg1(row + u + j * r.step), id, id, id};
      }
#pragma unroll
      for (int j = 0; j < U; ++j) acc = cop4<T, Op>(acc, v[j]);
    }
    for (; u < r.end; u += r.step) {
      if constexpr (VEC) acc = cop4<T, Op>(acc, ldg4(row + 4 * u));
      else acc.x = Op::apply(acc.x, ldg1(row + u));
    }
    T res;
    if (cluster_team_reduce<Op, CTA / 32>(Op::apply(Op::apply(acc.x, acc.y), Op::apply(acc.z, acc.w)),
                                          wsum, part, master_part, par, rank, started, &res))
      out[item] = init ? Op::apply(init[item], res) : res;  // the master finishes alone
  }
  if (!started) cluster_wait();
}

// ---------------------------------------------------------------- MV
// y[i] = sum_j A[i*lda+j] x[j] with a cluster per row: MV with few, long rows
// (the Fig 14 axis, taken to rows fewer than SMs).
template <int S, int DIST, bool VEC>
__global__ void __launch_bounds__(S / kClusterCtas, 4096 / S > 0 ? 4096 / S : 1)  // <= 128 registers
mv_cluster_kernel(const float* __restrict__ A, int64_t lda, const float* __restrict__ x,
                  float* __restrict__ y, int64_t h, int64_t w) {
  pdl_entry();
  constexpr int CTA = S / kClusterCtas;
  __shared__ float wsum[2 * (CTA / 32)];
  __shared__ float part[2][kClusterCtas];
  cg::cluster_group cluster = cg::this_cluster();
  const int rank = (int)cluster.block_rank();
  const int slave = rank * CTA + threadIdx.x;
  const int64_t nunits = VEC ? (w >> 2) : w;
  const Range<S, DIST> r(nunits, w, VEC ? 4 : 1, slave);
  const int64_t cid = blockIdx.x / kClusterCtas, ncl = gridDim.x / kClusterCtas;
  float* master_part = cluster.map_shared_rank(&part[0][0], 0);
  cluster_arrive_relaxed();
  bool started = false;
  int par = 0;
  for (int64_t row = cid; row < h; row += ncl, par ^= 1) {
    const float* a = A + row * lda;
    V4<float> acc = {0.f, 0.f, 0.f, 0.f};
    int64_t u = r.begin;
    constexpr int U = 4;
    for (; u + (U - 1) * r.step < r.end; u += U * r.step) {
      V4<float> av[U], xv[U];
#pragma unroll
      for (int j = 0; j < U; ++j) {
        const int64_t uu = u + j * r.step;
        if constexpr (VEC) { av[j] = ldg4_stream(a + 4 * uu); xv[j] = ldg4(x + 4 * uu); }
        else { av[j] = {ldg1(a + uu), 0.f, 0.f, 0.f}; xv[j] = {ldg1(x + uu), 0.f, 0.f, 0.f}; }
      }
#pragma unroll
      for (int j = 0; j < U; ++j) {
        acc.x = fmaf(av[j].x, xv[j].x, acc.x);
        acc.y = fmaf(av[j].y, xv[j].y, acc.y);
        acc.z = fmaf(av[j].z, xv[j].z, acc.z);
        acc.w = fmaf(av[j].w, xv[j].w, acc.w);
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
    float res;
    if (cluster_team_reduce<OpSum, CTA / 32>((acc.x + acc.y) + (acc.z + acc.w), wsum, part, master_part,
                                             par, rank, started, &res))
      y[row] = res;
  }
  if (!started) cluster_wait();
}

// ---------------------------------------------------------------- batched scan (block)
// out[n*L+k] = init[n] + sum_{i<=k} in[n*L+i] with a cluster per item, block
// distribution (R5): pass 1 sums each slave's chunk; the CTA scans its
// threads' chunk sums (shfl per warp, shared memory across warps);
// each CTA publishes its total in its own shared memory and, after one
// cluster barrier, reads the totals of the lower ranks -- and the master
// CTA's carry-in init[n], a live-in broadcast over DSMEM --
// to get its offset; pass 2 re-reads the chunk and stores the running values
// (every team member stores its own elements).  Only the block
// distribution is built: a cyclic cluster-wide scan needs a cluster barrier
// per round of S units.
template <class T, int S, bool VEC>
__global__ void __launch_bounds__(S / kClusterCtas, 4096 / S > 0 ? 4096 / S : 1)
scan_cluster_kernel(const T* __restrict__ in, const T* __restrict__ init, T* __restrict__ out,
                    int64_t N, int64_t L) {
  pdl_entry();
  constexpr int CTA = S / kClusterCtas;
  constexpr int W = CTA / 32;
  constexpr int V = VEC ? 4 : 1;
  __shared__ T wsum[2][W];
  __shared__ T tot[2];    // this CTA's total (read by higher ranks over DSMEM)
  __shared__ T cin[2];    // the master CTA's carry-in (read by every rank)
  __shared__ T off[2];    // this CTA's offset
  cg::cluster_group cluster = cg::this_cluster();
  const int rank = (int)cluster.block_rank();
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int slave = rank * CTA + tid;
  const int64_t nunits = VEC ? (L >> 2) : L;
  const Range<S, DIST_BLOCK> r(nunits, L, V, slave);
  const int64_t cid = blockIdx.x / kClusterCtas, ncl = gridDim.x / kClusterCtas;
  cluster_arrive_relaxed();
  bool started = false;
  int par = 0;
  for (int64_t item = cid; item < N; item += ncl, par ^= 1) {
    const T* irow = in + item * L;
    T* orow = out + item * L;
    // pass 1: this slave's chunk sum (U loads in flight, then the adds)
    constexpr int U = 8;
    T csum = T(0);
    int64_t u = r.begin;
    for (; u + U <= r.end; u += U) {
      T v[U];
#pragma unroll
      for (int j = 0; j < U; ++j) {
        if constexpr (VEC) v[j] = sum4(ldg4(irow + 4 * (u + j)));
        else v[j] = ldg1(irow + u + j);
      }
#pragma unroll
      for (int j = 0; j < U; ++j) csum = OpSum::apply(csum, v[j]);
    }
    for (; u < r.end; ++u) {
      if constexpr (VEC) csum = OpSum::apply(csum, sum4(ldg4(irow + 4 * u)));
      else csum = OpSum::apply(csum, ldg1(irow + u));
    }
    // CTA-wide exclusive scan of the chunk sums
    T incl = csum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const T t = __shfl_up_sync(kFull, incl, o);
      if (lane >= o) incl = OpSum::apply(incl, t);
    }
    if (lane == 31) wsum[par][wid] = incl;
    if (!started) {  // CTA-uniform; see cluster_team_reduce
      cluster_wait();
      started = true;
    }
    __syncthreads();
    T wpre = T(0), ctot = T(0);
#pragma unroll 4
    for (int k = 0; k < W; ++k) {
      const T q = wsum[par][k];
      if (k < wid) wpre = OpSum::apply(wpre, q);
      ctot = OpSum::apply(ctot, q);
    }
    if (tid == 0) {
      tot[par] = ctot;
      if (rank == 0) cin[par] = init ? init[item] : T(0);  // the master's sequential section
    }
    cluster.sync();  // totals and carry-in visible cluster-wide
    if (wid == 0) {  // offset = carry-in + totals of the lower ranks, over DSMEM
      T v = T(0);
      if (lane < rank) v = *cluster.map_shared_rank(&tot[par], lane);
      if (lane == 31) v = *cluster.map_shared_rank(&cin[par], 0);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) v = OpSum::apply(v, __shfl_xor_sync(kFull, v, o));
      if (lane == 0) off[par] = v;
    }
    __syncthreads();
    // pass 2: rescan the chunk from this slave's offset and store
    T run = OpSum::apply(off[par], OpSum::apply(wpre, warp_prev(incl)));
    u = r.begin;
    for (; u + U <= r.end; u += U) {
      if constexpr (VEC) {
        V4<T> v[U];
#pragma unroll
        for (int j = 0; j < U; ++j) v[j] = ldg4(irow + 4 * (u + j));
#pragma unroll
        for (int j = 0; j < U; ++j) {
          v[j].x = OpSum::apply(run, v[j].x); v[j].y = OpSum::apply(v[j].x, v[j].y);
          v[j].z = OpSum::apply(v[j].y, v[j].z); v[j].w = OpSum::apply(v[j].z, v[j].w);
          stg4(orow + 4 * (u + j), v[j]);
          run = v[j].w;
        }
      } else {
        T v[U];
#pragma unroll
        for (int j = 0; j < U; ++j) v[j] = ldg1(irow + u + j);
#pragma unroll
        for (int j = 0; j < U; ++j) {
          run = OpSum::apply(run, v[j]);
          orow[u + j] = run;
        }
      }
    }
    for (; u < r.end; ++u) {
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
    // Slots [par] (own tot/cin read remotely, wsum, off) are rewritten two
    // items later, after the next cluster barrier.
  }
  if (!started) cluster_wait();
  // Other CTAs read this CTA's tot/cin after the last item's barrier: no CTA
  // may exit (and release its shared memory) before they are done.
  cluster.sync();
}

// ---------------------------------------------------------------- batched scan (cyclic)
// Cyclic distribution: unit u belongs to slave u mod S, so in round k
// (units k*S .. k*S+S-1) CTA `rank` owns the contiguous units
// k*S + rank*CTA + [0, CTA) -- every warp load is coalesced.  A unit's prefix
// needs every unit of the earlier rounds and of the lower ranks in its own
// round; instead of a cluster barrier per round, rounds are processed in
// chunks of RC rounds, two passes per chunk:
//   pass 1: each warp scans its units of every round of the chunk
//           (shfl-up) and keeps the warp totals wt[k][w] in shared
//           memory; the CTA totals tot[k] are published locally behind one
//           cluster barrier;
//   exchange: thread k reads the 8 CTAs' tot[k] (and the master
//           CTA's carry-in init[n], read_from_master one level up) and the
//           CTA turns them into the offset of each (round, warp) -- every CTA
//           computes the same chunk total, in the same order, for its carry;
//   pass 2: re-read the chunk (an L2 hit: RC = 16 rounds keep <= 256 KB per SM
//           in flight between the passes, 37 MB over the GPU; with 32 rounds
//           and 1024-thread CTAs ncu saw a 14 % L2 hit rate), local scan +
//           the same warp scan + offset, store.
// The warp totals come from the same shfl-up scan in both passes, so the
// offsets and the stored values agree bit for bit.
constexpr int kScanRC = 16;  // rounds per chunk: <= 256 KB of pass-1 data per SM stays in L2 for pass 2
constexpr int kScanG = 8;    // rounds whose loads are in flight together
// CUDANP_SCL_PF=1: pass 2's first group of loads (L2 hits) is issued before the
// cluster barrier, so its latency overlaps the barrier and the exchange.
// CUDANP_SCL_PF=2: also the next chunk's (or next item's) first pass-1 group is
// issued right after pass 2's last loads, under pass 2's scans and stores.
// A push exchange (st.async of the per-round totals into every CTA's shared
// memory, counted on mbarriers, instead of the cluster barrier) was measured
// at +5-9 % in round 1 but rejected: compute-sanitizer synccheck reported a
// divergent warp at the CTA barrier after the exchange.
// A/B (profiles/exp_sclpf_*_r01o.jsonl, 16 x 4M and 256 x 256K int32): PF=1
// +2-5 % on every cyclic cluster size, PF=2 up to -14 % (the 1024-thread CTAs'
// 64-register cap spills the second group), so PF=1 is the default.
#ifndef CUDANP_SCL_PF
#define CUDANP_SCL_PF 1
#endif

template <class T, int S, bool VEC>
__global__ void __launch_bounds__(S / kClusterCtas, 4096 / S > 0 ? 4096 / S : 1)
scan_cluster_cyclic_kernel(const T* __restrict__ in, const T* __restrict__ init,
                           T* __restrict__ out, int64_t N, int64_t L) {
  pdl_entry();
  constexpr int CTA = S / kClusterCtas;
  constexpr int W = CTA / 32;
  constexpr int RC = kScanRC;
  constexpr int G = kScanG;
  static_assert(RC % G == 0, "whole groups per chunk");
  static_assert(RC <= 32 && RC * W <= CTA, "one lane per round / per (round, warp)");
  __shared__ T wt[RC][W];        // warp totals of the chunk's rounds (pass 1)
  __shared__ T offw[RC][W];      // offset of each (round, warp)
  __shared__ T tot[2][RC];       // this CTA's per-round totals (read over DSMEM)
  __shared__ T cin[2];           // the master CTA's carry-in
  __shared__ T carry_s;
  cg::cluster_group cluster = cg::this_cluster();
  const int rank = (int)cluster.block_rank();
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int64_t nunits = VEC ? (L >> 2) : L;
  const int64_t nrounds = (nunits + S - 1) / S;
  const int64_t cid = blockIdx.x / kClusterCtas, ncl = gridDim.x / kClusterCtas;
  cluster_arrive_relaxed();
  bool started = false;
  int par = 0;
  auto unit_load = [&](const T* row, int64_t u) -> V4<T> {
    V4<T> v = {T(0), T(0), T(0), T(0)};
    if (u < nunits) {
      if constexpr (VEC) v = ldg4(row + 4 * u);
      else v.x = ldg1(row + u);
    }
    return v;
  };
  auto warp_incl = [&](T x) {
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const T t = __shfl_up_sync(kFull, x, o);
      if (lane >= o) x = OpSum::apply(x, t);
    }
    return x;
  };
  V4<T> nx[G];             // PF=2: the next chunk's first pass-1 group
  bool have_nx = false;
  for (int64_t item = cid; item < N; item += ncl) {
    const T* irow = in + item * L;
    T* orow = out + item * L;
    if (tid == 0) {
      if (rank == 0) cin[par] = init ? init[item] : T(0);  // the master's sequential section
      carry_s = T(0);
    }
    bool first = true;
    for (int64_t k0 = 0; k0 < nrounds; k0 += RC, par ^= 1) {
      const int rc = (int)(nrounds - k0 < RC ? nrounds - k0 : RC);
      // pass 1: warp totals per round (G rounds' loads in flight at a time)
      for (int kg = 0; kg < rc; kg += G) {
        V4<T> v[G];
        if (CUDANP_SCL_PF >= 2 && kg == 0 && have_nx) {
#pragma unroll
          for (int j = 0; j < G; ++j) v[j] = nx[j];
        } else {
#pragma unroll
          for (int j = 0; j < G; ++j) v[j] = unit_load(irow, (k0 + kg + j) * S + rank * CTA + tid);
        }
#pragma unroll
        for (int j = 0; j < G; ++j) {
          if (kg + j >= rc) break;
          const T ut = VEC ? OpSum::apply(OpSum::apply(OpSum::apply(v[j].x, v[j].y), v[j].z), v[j].w) : v[j].x;
          const T wi = warp_incl(ut);
          if (lane == 31) wt[kg + j][wid] = wi;
        }
      }
      V4<T> vv[G];
      if constexpr (CUDANP_SCL_PF) {
#pragma unroll
        for (int j = 0; j < G; ++j) vv[j] = unit_load(irow, (k0 + j) * S + rank * CTA + tid);
      }
      if (!started) {  // CTA-uniform; see cluster_team_reduce
        cluster_wait();
        started = true;
      }
      __syncthreads();
      if (tid < rc) {
        T c = wt[tid][0];
#pragma unroll
        for (int w = 1; w < W; ++w) c = OpSum::apply(c, wt[tid][w]);
        tot[par][tid] = c;
      }
      cluster.sync();  // every CTA's tot[par] (and the carry-in) visible cluster-wide
      // exchange: lane k of warp 0 gathers round k's totals of all ranks
      if (wid == 0) {
        T rowt = T(0), low = T(0);
        if (lane < rc) {
#pragma unroll
          for (int r = 0; r < kClusterCtas; ++r) {
            const T t = *cluster.map_shared_rank(&tot[par][lane], r);
            rowt = OpSum::apply(rowt, t);
            if (r < rank) low = OpSum::apply(low, t);
          }
        }
        const T incl = warp_incl(rowt);                   // rounds 0..k of the chunk
        const T chunk_total = __shfl_sync(kFull, incl, 31);
        T base = carry_s;
        if (first) base = OpSum::apply(base, *cluster.map_shared_rank(&cin[par], 0));
        // offset of round k for this CTA = base + rounds < k + lower ranks in round k
        const T offk = OpSum::apply(base, OpSum::apply(warp_prev(incl), low));
        if (lane < rc) {
          T o = offk;
#pragma unroll
          for (int w = 0; w < W; ++w) {
            offw[lane][w] = o;
            o = OpSum::apply(o, wt[lane][w]);
          }
        }
        __syncwarp();
        if (lane == 0) carry_s = OpSum::apply(base, chunk_total);
      }
      first = false;
      __syncthreads();
      // pass 2: rescan and store
      for (int kg = 0; kg < rc; kg += G) {
        if (!CUDANP_SCL_PF || kg > 0) {
#pragma unroll
          for (int j = 0; j < G; ++j) vv[j] = unit_load(irow, (k0 + kg + j) * S + rank * CTA + tid);
        }
        if (CUDANP_SCL_PF >= 2 && kg + G >= rc) {  // last group: issue the next chunk's first loads
          const bool same = k0 + RC < nrounds;
          const int64_t nitem = same ? item : item + ncl;
          const int64_t nk0 = same ? k0 + RC : 0;
          have_nx = nitem < N;
          if (have_nx) {
            const T* nrow = in + nitem * L;
#pragma unroll
            for (int j = 0; j < G; ++j) nx[j] = unit_load(nrow, (nk0 + j) * S + rank * CTA + tid);
          }
        }
#pragma unroll
        for (int j = 0; j < G; ++j) {
          if (kg + j >= rc) break;
          const int64_t u = (k0 + kg + j) * S + rank * CTA + tid;
          V4<T> v = vv[j];
          if constexpr (VEC) {
            v.y = OpSum::apply(v.x, v.y); v.z = OpSum::apply(v.y, v.z); v.w = OpSum::apply(v.z, v.w);
          }
          const T ut = VEC ? v.w : v.x;
          const T wi = warp_incl(ut);
          const T add = OpSum::apply(offw[kg + j][wid], warp_prev(wi));
          if (u < nunits) {
            if constexpr (VEC)
              stg4(orow + 4 * u, V4<T>{OpSum::apply(add, v.x), OpSum::apply(add, v.y),
                                       OpSum::apply(add, v.z), OpSum::apply(add, v.w)});
            else orow[u] = OpSum::apply(add, v.x);
          }
        }
      }
      __syncthreads();  // wt / offw / carry_s reused by the next chunk
    }
  }
  if (!started) cluster_wait();
  cluster.sync();  // remote reads of tot/cin are done before any CTA exits
}

#define CUDANP_DISPATCH_CLUSTER_S(S, ...)                      \
  switch (S) {                                                 \
    case 2048: { constexpr int kS = 2048; __VA_ARGS__; } break; \
    case 4096: { constexpr int kS = 4096; __VA_ARGS__; } break; \
    case 8192: { constexpr int kS = 8192; __VA_ARGS__; } break; \
    default: return fail_invalid("S must be 2048, 4096 or 8192 for a cluster team"); \
  }

template <typename... KArgs, typename... Args>
static int launch_cluster(void (*kern)(KArgs...), int cta, int64_t N, cudaStream_t st,
                          LaunchInfo* info, const char* what, Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.blockDim = dim3(cta);
  cfg.dynamicSmemBytes = 0;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = kClusterCtas;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  // One cluster per item, up to 8 waves of resident clusters (the block
  // scheduler balances the small CTAs); then clusters stride over items.
  int resident = 0;
  cfg.gridDim = dim3(kClusterCtas);
  if (cudaOccupancyMaxActiveClusters(&resident, (void*)kern, &cfg) != cudaSuccess || resident < 1) {
    // No 8-CTA cluster of this kernel can be co-scheduled here (e.g. an MPS
    // SM limit or a MIG slice): a valid team size this device cannot run.
    cudaGetLastError();
    set_error("%s: no cluster of %d CTAs x %d threads can be resident on this device", what,
              kClusterCtas, cta);
    return CUDANP_ERR_UNSUPPORTED;
  }
  int64_t clusters = N < (int64_t)resident * 8 ? N : (int64_t)resident * 8;
  if (clusters < 1) clusters = 1;
  if (info) {
    info->block_threads = cta; info->grid = clusters * kClusterCtas; info->map = MAP_INTRA;
    kernel_attrs(kern, &info->regs, &info->smem);
    return CUDANP_OK;
  }
  if (N == 0) return CUDANP_OK;
  cfg.gridDim = dim3((unsigned)(clusters * kClusterCtas));
  cudaError_t e = cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
  if (e != cudaSuccess) {
    set_error("%s: %s", what, cudaGetErrorString(e));
    cudaGetLastError();
    return CUDANP_ERR_CUDA;
  }
  return check_launch(what);
}

template <class T, class Op>
static int reduce_cluster_t(const void* in, const void* init, void* out, int64_t N, int64_t L,
                            int S, int dist, bool vec, cudaStream_t st, LaunchInfo* info) {
  CUDANP_DISPATCH_CLUSTER_S(S, {
    constexpr int CTA = kS / kClusterCtas;
    void (*kern)(const T*, const T*, T*, int64_t, int64_t) =
        dist == DIST_CYCLIC
            ? (vec ? reduce_cluster_kernel<T, Op, kS, DIST_CYCLIC, true> : reduce_cluster_kernel<T, Op, kS, DIST_CYCLIC, false>)
            : (vec ? reduce_cluster_kernel<T, Op, kS, DIST_BLOCK, true> : reduce_cluster_kernel<T, Op, kS, DIST_BLOCK, false>);
    return launch_cluster(kern, CTA, N, st, info, "batched_loop_reduce (cluster team) launch",
                          (const T*)in, (const T*)init, (T*)out, N, L);
  });
  return CUDANP_OK;
}

int reduce_cluster(const void* in, const void* init, void* out, int64_t N, int64_t L, int dtype,
                   int op, int S, int dist, bool vec, cudaStream_t st, LaunchInfo* info) {
  if (dtype == CUDANP_F32)
    return op == CUDANP_SUM ? reduce_cluster_t<float, OpSum>(in, init, out, N, L, S, dist, vec, st, info)
                            : reduce_cluster_t<float, OpMax>(in, init, out, N, L, S, dist, vec, st, info);
  return op == CUDANP_SUM ? reduce_cluster_t<int32_t, OpSum>(in, init, out, N, L, S, dist, vec, st, info)
                          : reduce_cluster_t<int32_t, OpMax>(in, init, out, N, L, S, dist, vec, st, info);
}

int mv_cluster(const float* A, int64_t lda, const float* x, float* y, int64_t h, int64_t w, int S,
               int dist, bool vec, cudaStream_t st, LaunchInfo* info) {
  CUDANP_DISPATCH_CLUSTER_S(S, {
    constexpr int CTA = kS / kClusterCtas;
    auto kern = dist == DIST_CYCLIC ? (vec ? mv_cluster_kernel<kS, DIST_CYCLIC, true> : mv_cluster_kernel<kS, DIST_CYCLIC, false>)
                                    : (vec ? mv_cluster_kernel<kS, DIST_BLOCK, true> : mv_cluster_kernel<kS, DIST_BLOCK, false>);
    return launch_cluster(kern, CTA, h, st, info, "mv (cluster team) launch", A, lda, x, y, h, w);
  });
  return CUDANP_OK;
}

template <class T>
static int scan_cluster_t(const void* in, const void* init, void* out, int64_t N, int64_t L, int S,
                          int dist, bool vec, cudaStream_t st, LaunchInfo* info) {
  CUDANP_DISPATCH_CLUSTER_S(S, {
    constexpr int CTA = kS / kClusterCtas;
    auto kern = dist == DIST_CYCLIC
                    ? (vec ? scan_cluster_cyclic_kernel<T, kS, true> : scan_cluster_cyclic_kernel<T, kS, false>)
                    : (vec ? scan_cluster_kernel<T, kS, true> : scan_cluster_kernel<T, kS, false>);
    if (!info && (N == 0 || L == 0)) return CUDANP_OK;
    return launch_cluster(kern, CTA, N, st, info, "batched_loop_scan (cluster team) launch",
                          (const T*)in, (const T*)init, (T*)out, N, L);
  });
  return CUDANP_OK;
}

int scan_cluster(const void* in, const void* init, void* out, int64_t N, int64_t L, int dtype, int S,
                 int dist, bool vec, cudaStream_t st, LaunchInfo* info) {
  return dtype == CUDANP_F32 ? scan_cluster_t<float>(in, init, out, N, L, S, dist, vec, st, info)
                             : scan_cluster_t<int32_t>(in, init, out, N, L, S, dist, vec, st, info);
}

}  // namespace cudanp
