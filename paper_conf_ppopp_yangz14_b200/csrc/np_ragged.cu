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
#define CUDANP_RAGGED_K 2
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

// One slave's view of a segment [b, b+len): head (< 4 scalars up to the next
// 16-byte boundary), aligned body of nu 128-bit units dealt over the team by
// the distribution, tail (< 4 scalars).  All index math is done once per item
// and the body walks a pointer; per-element 64-bit arithmetic made the first
// version instruction-bound (ncu: 4 B per warp instruction).
template <class T, int S, int DIST>
struct SegShare {
  const T* body;      // this slave's first body unit
  int64_t step;       // elements between its consecutive units
  int cnt;            // body units it owns
  int head, tail;     // segment head/tail lengths
  __device__ __forceinline__ SegShare(const T* in, int64_t b, int64_t len, int slave) {
    const int mis = (int)(((uintptr_t)(in + b) >> 2) & 3);  // elements past a 16-byte line
    int64_t h = (4 - mis) & 3;
    if (h > len) h = len;
    const int64_t nu = (len - h) >> 2;
    head = (int)h;
    tail = (int)(len - h - 4 * nu);
    const Range<S, DIST> r(nu, 4 * nu, 4, slave);
    cnt = r.end > r.begin ? (int)((r.end - r.begin + r.step - 1) / r.step) : 0;
    body = in + b + h + 4 * r.begin;
    step = 4 * r.step;
  }
};

// ---------------------------------------------------------------- intra-warp
// K consecutive warp tiles per warp step.  The step is written in three
// phases so that nothing waits on a round trip it does not need: (1) the
// masters' sequential sections for all K items issue their bound loads
// together; (2) the bounds are broadcast and every slave works
// out its share; (3) all head/tail scalars and the body's first units are in
// flight before the first use.  A per-item version (load bounds, shfl, load
// head, ...) paid K dependent round trips per step and ran short segments at
// a third of the tuned S=1 rate.
//
// UNI: every item has the same trip count L and starts at n*L (the batched
// reduce when its rows are not 16-byte aligned, L % 4 != 0): the bounds are
// uniform index math, recomputed by every slave instead of loaded and
// broadcast, and the same head/body/tail peeling gives each row
// 128-bit body loads.
template <class T, class Op, int S, int DIST, int KT = kRaggedK, bool UNI = false>
__global__ void __launch_bounds__(kRaggedBlock)
ragged_intra_kernel(const T* __restrict__ in, const int64_t* __restrict__ off,
                    const T* __restrict__ init, T* __restrict__ out, int64_t N, int64_t L) {
  pdl_entry();
  constexpr int TPW = 32 / S;
  constexpr int K = KT;
  constexpr int HM = (3 + S - 1) / S;  // head (or tail) scalars per slave, at most
  const IntraTeam<S> team;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t ntiles = (N + TPW - 1) / TPW;
  const T id = Op::template identity<T>();

  for (int64_t t0 = warp * K; t0 < ntiles; t0 += nwarps * K) {
    int64_t item[K], b[K], e[K];
    // (1) Sequential section (master only): read the loop bounds.
#pragma unroll
    for (int k = 0; k < K; ++k) {
      item[k] = (t0 + k) * TPW + team.team;
      b[k] = 0; e[k] = 0;
      if (UNI) {
        if (item[k] < N) { b[k] = item[k] * L; e[k] = b[k] + L; }
      } else if (team.is_master() && item[k] < N) {
        b[k] = off[item[k]];
        e[k] = off[item[k] + 1];
      }
    }
    const T* p[K];
    int64_t pstep[K];
    int cnt[K];
    T part[K];
    int trips = 0;
#pragma unroll
    for (int k = 0; k < K; ++k) {
      // (2) ... broadcast them to the slaves.
      const int64_t bk = UNI ? b[k] : team.read_from_master(b[k]);
      int64_t len = (UNI ? e[k] : team.read_from_master(e[k])) - bk;
      if (len < 0) len = 0;  // a decreasing offset pair is an empty loop
      const SegShare<T, S, DIST> sh(in, bk, len, team.slave);
      p[k] = sh.body;
      pstep[k] = sh.step;
      cnt[k] = sh.cnt;
      trips = max(trips, sh.cnt);
      // (3) head and tail scalars (< 4 each), dealt over the first slaves
      const T* tl = in + bk + sh.head + 4 * ((len - sh.head) >> 2);
      T hv[HM], tv[HM];
#pragma unroll
      for (int j = 0; j < HM; ++j) {
        const int i = team.slave + j * S;
        hv[j] = i < sh.head ? ldg1(in + bk + i) : id;
        tv[j] = i < sh.tail ? ldg1(tl + i) : id;
      }
      part[k] = id;
#pragma unroll
      for (int j = 0; j < HM; ++j) part[k] = Op::apply(part[k], Op::apply(hv[j], tv[j]));
    }
    trips = (int)__reduce_max_sync(kFull, (unsigned)trips);  // warp-uniform trip count
    V4<T> acc[K];
#pragma unroll
    for (int k = 0; k < K; ++k) acc[k] = {id, id, id, id};
#pragma unroll kRaggedUnroll
    for (int j = 0; j < trips; ++j) {
      V4<T> v[K];
#pragma unroll
      for (int k = 0; k < K; ++k) {
        if (j < cnt[k]) v[k] = ldg4(p[k]);
        else v[k] = {id, id, id, id};
        p[k] += pstep[k];
      }
#pragma unroll
      for (int k = 0; k < K; ++k) acc[k] = op4r<T, Op>(acc[k], v[k]);
    }
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const T pk = Op::apply(part[k], Op::apply(Op::apply(acc[k].x, acc[k].y), Op::apply(acc[k].z, acc[k].w)));
      const T res = team.template reduce<Op>(pk);
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
  __shared__ int64_t slot_b[32], slot_l[32];
  __shared__ T red[S][33];
  const InterTeam<S> team;
  const int64_t ngroups = (N + 31) / 32;
  const T id = Op::template identity<T>();
  for (int64_t g = blockIdx.x; g < ngroups; g += gridDim.x) {
    const int64_t item = g * 32 + team.master;
    const bool ok = item < N;
    int64_t b0 = 0, l0 = 0;
    if (team.is_master() && ok) {
      b0 = off[item];
      l0 = off[item + 1] - b0;
      if (l0 < 0) l0 = 0;
    }
    team.read_from_master(b0, l0, slot_b, slot_l);
    const int64_t b = b0, len = l0;
    const SegShare<T, S, DIST> sh(in, b, len, team.slave);
    T pv = id;
    for (int i = team.slave; i < sh.head; i += S) pv = Op::apply(pv, in[b + i]);
    const T* tl = in + b + sh.head + 4 * ((len - sh.head) >> 2);
    for (int i = team.slave; i < sh.tail; i += S) pv = Op::apply(pv, tl[i]);
    V4<T> acc = {id, id, id, id};
    const T* q = sh.body;
    int c = 0;
    for (; c + 4 <= sh.cnt; c += 4, q += 4 * sh.step) {  // 4 loads in flight, then fold
      V4<T> v[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) v[j] = ldg4(q + j * sh.step);
#pragma unroll
      for (int j = 0; j < 4; ++j) acc = op4r<T, Op>(acc, v[j]);
    }
    for (; c < sh.cnt; ++c, q += sh.step) acc = op4r<T, Op>(acc, ldg4(q));
    pv = Op::apply(pv, Op::apply(Op::apply(acc.x, acc.y), Op::apply(acc.z, acc.w)));
    if (S == 1) {
      if (ok) out[item] = init ? Op::apply(init[item], pv) : pv;
      continue;
    }
    red[team.slave][team.master] = pv;
    __syncthreads();
    if (team.is_master() && ok) {
      T res = red[0][team.master];
#pragma unroll
      for (int s2 = 1; s2 < S; ++s2) res = Op::apply(res, red[s2][team.master]);
      out[item] = init ? Op::apply(init[item], res) : res;
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------- multi-warp team (S > 32)
// Few, long segments: a team of S/32 consecutive warps per segment (shfl per
// warp + shared memory across them); bounds broadcast through a shared slot.
template <class T, class Op, int S, int DIST>
__global__ void __launch_bounds__(MultiShape<S>::CTA, MultiShape<S>::MINB)
ragged_multi_kernel(const T* __restrict__ in, const int64_t* __restrict__ off,
                    const T* __restrict__ init, T* __restrict__ out, int64_t N) {
  using Sh = MultiShape<S>;
  __shared__ T sm[Sh::TEAMS * MultiTeam<S>::W];
  __shared__ int64_t slot_b[Sh::TEAMS], slot_l[Sh::TEAMS];
  const MultiTeam<S> team;
  const int64_t ngroups = (N + Sh::TEAMS - 1) / Sh::TEAMS;
  const T id = Op::template identity<T>();
  for (int64_t g = blockIdx.x; g < ngroups; g += gridDim.x) {
    const int64_t item = g * Sh::TEAMS + team.team;
    const bool ok = item < N;
    int64_t b0 = 0, l0 = 0;
    if (team.is_master() && ok) {  // sequential section: the master reads the bounds
      b0 = off[item];
      l0 = off[item + 1] - b0;
      if (l0 < 0) l0 = 0;
    }
    const int64_t b = team.read_from_master(b0, slot_b);
    const int64_t len = team.read_from_master(l0, slot_l);
    const SegShare<T, S, DIST> sh(in, b, len, team.slave);
    T pv = id;
    for (int i = team.slave; i < sh.head; i += S) pv = Op::apply(pv, in[b + i]);
    const T* tl = in + b + sh.head + 4 * ((len - sh.head) >> 2);
    for (int i = team.slave; i < sh.tail; i += S) pv = Op::apply(pv, tl[i]);
    V4<T> acc = {id, id, id, id};
    const T* q = sh.body;
    int c = 0;
    for (; c + 4 <= sh.cnt; c += 4, q += 4 * sh.step) {
      V4<T> v[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) v[j] = ldg4(q + j * sh.step);
#pragma unroll
      for (int j = 0; j < 4; ++j) acc = op4r<T, Op>(acc, v[j]);
    }
    for (; c < sh.cnt; ++c, q += sh.step) acc = op4r<T, Op>(acc, ldg4(q));
    pv = Op::apply(pv, Op::apply(Op::apply(acc.x, acc.y), Op::apply(acc.z, acc.w)));
    const T res = team.template reduce<Op>(pv, sm);
    if (team.is_master() && ok) out[item] = init ? Op::apply(init[item], res) : res;
  }
}

template <class T, class Op>
static int launch_ragged_multi(const T* in, const int64_t* off, const T* init, T* out, int64_t N,
                               int S, int dist, cudaStream_t st) {
#define CUDANP_RAGGED_BIG(SV)                                                                     \
  case SV: {                                                                                      \
    auto kern = dist == DIST_CYCLIC ? ragged_multi_kernel<T, Op, SV, DIST_CYCLIC>                 \
                                    : ragged_multi_kernel<T, Op, SV, DIST_BLOCK>;                 \
    using Sh = MultiShape<SV>;                                                                    \
    const int64_t grid = persistent_grid(kern, Sh::CTA, 0, (N + Sh::TEAMS - 1) / Sh::TEAMS);      \
    kern<<<(unsigned)grid, Sh::CTA, 0, st>>>(in, off, init, out, N);                              \
    return check_launch("ragged_loop_reduce (multi-warp team) launch");                          \
  }
  switch (S) {
    CUDANP_RAGGED_BIG(64) CUDANP_RAGGED_BIG(128) CUDANP_RAGGED_BIG(256) CUDANP_RAGGED_BIG(512)
    CUDANP_RAGGED_BIG(1024)
    default: return fail_invalid("S");
  }
#undef CUDANP_RAGGED_BIG
}

// ---------------------------------------------------------------- adaptive team size
// Segment lengths vary (exponential mixes, P:340's imbalance): a fixed S
// either wastes slaves on short segments or leaves long ones to one thread.
// Here the team size is chosen per segment at run time, the way the master
// decides in its sequential section whether to wake its slaves for a loop
// whose bound it has just read: each lane is the master of one
// segment of the warp's 32; segments shorter than `thresh` are run by their
// master alone (S = 1, 128-bit body units), and each longer one is run by
// the whole warp as a team of 32 (cyclic units), the masters taking
// turns (ballot of the long ones, bounds broadcast by shfl from their
// master), with a butterfly team reduction; the master stores
// (P:327).  Every segment is still reduced by exactly one team.
template <class T, class Op>
__global__ void __launch_bounds__(kRaggedBlock)
ragged_adaptive_kernel(const T* __restrict__ in, const int64_t* __restrict__ off,
                       const T* __restrict__ init, T* __restrict__ out, int64_t N, int64_t thresh) {
  pdl_entry();
  constexpr int K = 2;  // tiles of 32 segments per warp step: their bound loads overlap
  const int lane = threadIdx.x & 31;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t ntiles = (N + 31) / 32;
  const T id = Op::template identity<T>();
  for (int64_t t0 = warp * K; t0 < ntiles; t0 += nwarps * K) {
    int64_t item[K], b[K], len[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {  // sequential sections: each master reads its loop bounds
      item[k] = (t0 + k) * 32 + lane;
      b[k] = 0; len[k] = 0;
      if (item[k] < N) {
        b[k] = off[item[k]];
        len[k] = off[item[k] + 1] - b[k];
        if (len[k] < 0) len[k] = 0;
      }
    }
    T part[K];
    // short segments: each master alone (a team of one); all K items' loads in flight
    {
      const T* p[K];
      int cnt[K];
      int64_t stp[K];
      int trips = 0;
#pragma unroll
      for (int k = 0; k < K; ++k) {
        const int64_t ls = len[k] >= thresh ? 0 : len[k];
        const SegShare<T, 1, DIST_CYCLIC> sh(in, b[k], ls, 0);
        p[k] = sh.body; cnt[k] = sh.cnt; stp[k] = sh.step;
        trips = max(trips, sh.cnt);
        T hv[3], tv[3];
        const T* tl = in + b[k] + sh.head + 4 * ((ls - sh.head) >> 2);
#pragma unroll
        for (int j = 0; j < 3; ++j) {
          hv[j] = j < sh.head ? ldg1(in + b[k] + j) : id;
          tv[j] = j < sh.tail ? ldg1(tl + j) : id;
        }
        part[k] = Op::apply(Op::apply(Op::apply(hv[0], hv[1]), hv[2]), Op::apply(Op::apply(tv[0], tv[1]), tv[2]));
      }
      V4<T> acc[K];
#pragma unroll
      for (int k = 0; k < K; ++k) acc[k] = {id, id, id, id};
#pragma unroll 2
      for (int j = 0; j < trips; ++j) {
        V4<T> v[K];
#pragma unroll
        for (int k = 0; k < K; ++k) {
          v[k] = j < cnt[k] ? ldg4(p[k]) : V4<T>{id, id, id, id};
          p[k] += stp[k];
        }
#pragma unroll
        for (int k = 0; k < K; ++k) acc[k] = op4r<T, Op>(acc[k], v[k]);
      }
#pragma unroll
      for (int k = 0; k < K; ++k)
        part[k] = Op::apply(part[k], Op::apply(Op::apply(acc[k].x, acc[k].y), Op::apply(acc[k].z, acc[k].w)));
    }
    // long segments: the whole warp as one team, masters taking turns
#pragma unroll
    for (int k = 0; k < K; ++k) {
      unsigned m = __ballot_sync(kFull, len[k] >= thresh);
      while (m) {
        const int src = __ffs(m) - 1;
        m &= m - 1;
        const int64_t bb = __shfl_sync(kFull, b[k], src);   // read_from_master
        const int64_t ll = __shfl_sync(kFull, len[k], src);
        const SegShare<T, 32, DIST_CYCLIC> sh(in, bb, ll, lane);
        T pv = id;
        if (lane < sh.head) pv = Op::apply(pv, ldg1(in + bb + lane));
        const T* tl = in + bb + sh.head + 4 * ((ll - sh.head) >> 2);
        if (lane < sh.tail) pv = Op::apply(pv, ldg1(tl + lane));
        V4<T> acc[4] = {{id, id, id, id}, {id, id, id, id}, {id, id, id, id}, {id, id, id, id}};
        const T* p = sh.body;
        int c = 0;
        for (; c + 3 < sh.cnt; c += 4, p += 4 * sh.step) {
          V4<T> v[4];
#pragma unroll
          for (int j = 0; j < 4; ++j) v[j] = ldg4(p + j * sh.step);
#pragma unroll
          for (int j = 0; j < 4; ++j) acc[j] = op4r<T, Op>(acc[j], v[j]);
        }
        for (; c < sh.cnt; ++c, p += sh.step) acc[0] = op4r<T, Op>(acc[0], ldg4(p));
        const V4<T> a4 = op4r<T, Op>(op4r<T, Op>(acc[0], acc[1]), op4r<T, Op>(acc[2], acc[3]));
        pv = Op::apply(pv, Op::apply(Op::apply(a4.x, a4.y), Op::apply(a4.z, a4.w)));
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) pv = Op::apply(pv, __shfl_xor_sync(kFull, pv, o));
        if (lane == src) part[k] = pv;
      }
      if (item[k] < N) out[item[k]] = init ? Op::apply(init[item[k]], part[k]) : part[k];
    }
  }
}

template <class T, class Op>
static int launch_ragged_adaptive(const T* in, const int64_t* off, const T* init, T* out, int64_t N,
                                  int64_t thresh, cudaStream_t st) {
  if (N == 0) return CUDANP_OK;
  auto kern = ragged_adaptive_kernel<T, Op>;
  const int64_t grid = persistent_grid(kern, kRaggedBlock, 0, (N + 2 * kRaggedBlock - 1) / (2 * kRaggedBlock));
  launch_pdl(kern, dim3((unsigned)grid), dim3(kRaggedBlock), 0, st, in, off, init, out, N, thresh);
  return check_launch("ragged_loop_reduce (adaptive teams) launch");
}

int ragged_adaptive(const void* in, const int64_t* off, const void* init, void* out, int64_t N,
                    int dtype, int op, int64_t thresh, cudaStream_t st) {
  if (dtype == CUDANP_F32)
    return op == CUDANP_SUM
               ? launch_ragged_adaptive<float, OpSum>((const float*)in, off, (const float*)init, (float*)out, N, thresh, st)
               : launch_ragged_adaptive<float, OpMax>((const float*)in, off, (const float*)init, (float*)out, N, thresh, st);
  return op == CUDANP_SUM
             ? launch_ragged_adaptive<int32_t, OpSum>((const int32_t*)in, off, (const int32_t*)init, (int32_t*)out, N, thresh, st)
             : launch_ragged_adaptive<int32_t, OpMax>((const int32_t*)in, off, (const int32_t*)init, (int32_t*)out, N, thresh, st);
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
    constexpr int TPW = 32 / S;
    const int64_t ntiles = (N + TPW - 1) / TPW;
    const bool few = few_tiles(ragged_intra_kernel<T, Op, S, DIST>, kRaggedBlock, ntiles, kRaggedK);
    auto kern = few ? ragged_intra_kernel<T, Op, S, DIST, 1> : ragged_intra_kernel<T, Op, S, DIST, kRaggedK>;
    const int64_t per_cta = (kRaggedBlock / 32) * (few ? 1 : kRaggedK);
    const int64_t grid = persistent_grid(kern, kRaggedBlock, 0, (ntiles + per_cta - 1) / per_cta);
    launch_pdl(kern, dim3((unsigned)grid), dim3(kRaggedBlock), 0, st, in, off, init, out, N, (int64_t)-1);
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
  if (S > 32) {
    if (map == MAP_INTER) {
      set_error("a team of S > 32 is S/32 consecutive warps: intra-warp (consecutive) map only");
      return CUDANP_ERR_UNSUPPORTED;
    }
    if (N == 0) return CUDANP_OK;
    return launch_ragged_multi<T, Op>(i, off, ini, o, N, S, dist, st);
  }
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

// Batched reduce with rows that are not 16-byte aligned (L % 4 != 0 or a
// misaligned base): the UNI form of the intra-warp kernel above.
template <class T, class Op, int S, int DIST>
static int launch_uniform_peel(const T* in, const T* init, T* out, int64_t N, int64_t L,
                               cudaStream_t st, LaunchInfo* info) {
  constexpr int TPW = 32 / S;
  const int64_t ntiles = (N + TPW - 1) / TPW;
  const bool few = few_tiles(ragged_intra_kernel<T, Op, S, DIST, kRaggedK, true>, kRaggedBlock, ntiles, kRaggedK);
  auto kern = few ? ragged_intra_kernel<T, Op, S, DIST, 1, true> : ragged_intra_kernel<T, Op, S, DIST, kRaggedK, true>;
  const int64_t per_cta = (kRaggedBlock / 32) * (few ? 1 : kRaggedK);
  const int64_t grid = persistent_grid(kern, kRaggedBlock, 0, (ntiles + per_cta - 1) / per_cta);
  if (info) {
    info->block_threads = kRaggedBlock; info->grid = grid; info->map = MAP_INTRA;
    kernel_attrs(kern, &info->regs, &info->smem);
    return CUDANP_OK;
  }
  if (N == 0) return CUDANP_OK;
  launch_pdl(kern, dim3((unsigned)grid), dim3(kRaggedBlock), 0, st, in, (const int64_t*)nullptr, init, out, N, L);
  return check_launch("batched_loop_reduce (peeled rows) launch");
}

template <class T, class Op>
static int uniform_peel_t(const void* in, const void* init, void* out, int64_t N, int64_t L, int S,
                          int dist, cudaStream_t st, LaunchInfo* info) {
  const T* i = (const T*)in;
  const T* ini = (const T*)init;
  T* o = (T*)out;
  CUDANP_DISPATCH_S(S, {
    return dist == DIST_CYCLIC ? launch_uniform_peel<T, Op, kS, DIST_CYCLIC>(i, ini, o, N, L, st, info)
                               : launch_uniform_peel<T, Op, kS, DIST_BLOCK>(i, ini, o, N, L, st, info);
  });
  return CUDANP_OK;
}

int reduce_uniform_peel(const void* in, const void* init, void* out, int64_t N, int64_t L, int dtype,
                        int op, int S, int dist, cudaStream_t st, LaunchInfo* info) {
  if (dtype == CUDANP_F32)
    return op == CUDANP_SUM ? uniform_peel_t<float, OpSum>(in, init, out, N, L, S, dist, st, info)
                            : uniform_peel_t<float, OpMax>(in, init, out, N, L, S, dist, st, info);
  return op == CUDANP_SUM ? uniform_peel_t<int32_t, OpSum>(in, init, out, N, L, S, dist, st, info)
                          : uniform_peel_t<int32_t, OpMax>(in, init, out, N, L, S, dist, st, info);
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
