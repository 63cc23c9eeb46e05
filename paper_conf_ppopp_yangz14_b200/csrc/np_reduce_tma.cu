// np_reduce_tma.cu -- batched loop-reduce with the loop body staged by TMA:
// out[n] = init[n] (op) fold_i in[n*L+i]  (Fig 6d).
//
// Same method as reduce_intra_kernel (np_reduce.cu): an item's team is S
// consecutive lanes (intra-warp), each lane folds its share of the
// item's loop (cyclic P:166 / block R5) in 4-element units, the team combines
// the partials with the shfl butterfly and the master alone applies
// init[n] and stores.  The per-lane order of operations is the
// LDG kernel's, so both produce bit-identical results.
//
// What changes is how the item-major rows reach the team.  Items are
// contiguous, so a run of `ips` consecutive items is ONE contiguous block of
// ips*L*4 bytes: a producer warp streams such blocks with 1-D bulk copies
// (cp.async.bulk, completion counted on the stage's mbarrier) into a ring of
// shared-memory stages; sixteen consumer warps run the teams out of shared
// memory (K = 4 warp tiles in flight each) and release the stage.  The
// in-flight bytes then come from the ring (a few 32-64 KB stages per SM)
// rather than from resident warps and unrolled loads.
// Teams also make the shared-memory reads conflict-free: with the cyclic
// distribution a warp reads 32 consecutive 16-byte units.
#include "common.cuh"
#include "np_team.cuh"
#include "np_tma.cuh"

namespace cudanp {

#ifndef CUDANP_RT_WARPS
#define CUDANP_RT_WARPS 16
#endif
#ifndef CUDANP_RT_K
#define CUDANP_RT_K 4
#endif
constexpr int kRtWarps = CUDANP_RT_WARPS;         // consumer warps per CTA
constexpr int kRtThreads = 32 * (kRtWarps + 1);   // + one producer warp
constexpr int kRtK = CUDANP_RT_K;                 // warp tiles per consumer step (ILP)

template <class T, class Op>
__device__ __forceinline__ V4<T> rt_op4(V4<T> a, V4<T> b) {
  return {Op::apply(a.x, b.x), Op::apply(a.y, b.y), Op::apply(a.z, b.z), Op::apply(a.w, b.w)};
}

static __host__ __device__ __forceinline__ size_t rt_header_bytes(int stages) {
  return 128 * ((16 * (size_t)stages + 127) / 128);
}

template <class T, class Op, int S, int DIST>
__global__ void __launch_bounds__(kRtThreads, 1)
reduce_tma_kernel(const T* __restrict__ in, const T* __restrict__ init, T* __restrict__ out,
                  int64_t N, int64_t L, int ips, int stages) {
  pdl_entry();
  extern __shared__ __align__(128) unsigned char smem_raw[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw);
  uint64_t* empty = full + stages;
  T* ring = reinterpret_cast<T*>(smem_raw + rt_header_bytes(stages));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t nchunks = (N + ips - 1) / ips;
  const int64_t stage_elems = (int64_t)ips * L;
  // this CTA's chunks: blockIdx.x, blockIdx.x + gridDim.x, ...
  const int64_t mine = (int64_t)blockIdx.x < nchunks ? (nchunks - 1 - blockIdx.x) / gridDim.x + 1 : 0;

  if (threadIdx.x == 0) {
    for (int i = 0; i < stages; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], kRtWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  if (warp == kRtWarps) {
    // ---- producer warp: one bulk copy of ips items per stage
    if (lane == 0) {
      for (int64_t t = 0; t < mine; ++t) {
        const int st = (int)(t % stages);
        if (t >= stages) mbar_wait(&empty[st], (uint32_t)((t / stages) - 1) & 1);
        const int64_t n0 = ((int64_t)blockIdx.x + t * gridDim.x) * ips;
        const int64_t cnt = N - n0 < ips ? N - n0 : ips;
        const uint32_t bytes = (uint32_t)(cnt * L * (int64_t)sizeof(T));
        mbar_expect_tx(&full[st], bytes);
        bulk_load_1d(ring + st * stage_elems, in + n0 * L, bytes, &full[st]);
      }
    }
    return;
  }

  // ---- consumer warps: the NP teams
  constexpr int TPW = 32 / S;
  const IntraTeam<S> team;
  const Range<S, DIST> r(L >> 2, L, 4, team.slave);  // uniform: recomputed by every slave
  const T id = Op::template identity<T>();
  for (int64_t t = 0; t < mine; ++t) {
    const int st = (int)(t % stages);
    const int64_t n0 = ((int64_t)blockIdx.x + t * gridDim.x) * ips;
    const int cnt = (int)(N - n0 < ips ? N - n0 : ips);
    mbar_wait(&full[st], (uint32_t)(t / stages) & 1);
    const T* base = ring + st * stage_elems;
    const int ntile = (cnt + TPW - 1) / TPW;
    // K warp tiles per step (tile0 + k*warps, so a short stage still spreads
    // over every warp): K independent items per team in
    // flight, so shared-memory and shuffle latencies overlap.
    for (int tile0 = warp; tile0 < ntile; tile0 += kRtWarps * kRtK) {
      int il[kRtK];
      const T* row[kRtK];
      V4<T> acc[kRtK];
#pragma unroll
      for (int k = 0; k < kRtK; ++k) {
        il[k] = (tile0 + k * kRtWarps) * TPW + team.team;
        row[k] = base + (int64_t)(il[k] < cnt ? il[k] : 0) * L;
        acc[k] = {id, id, id, id};
      }
      // parallel loop section: the slave's units of each item (P:166 / R5)
      for (int64_t u = r.begin; u < r.end; u += r.step) {
#pragma unroll
        for (int k = 0; k < kRtK; ++k)
          acc[k] = rt_op4<T, Op>(acc[k], *reinterpret_cast<const V4<T>*>(row[k] + 4 * u));
      }
#pragma unroll
      for (int k = 0; k < kRtK; ++k) {
        const T part = Op::apply(Op::apply(acc[k].x, acc[k].y), Op::apply(acc[k].z, acc[k].w));
        const T res = team.template reduce<Op>(part);
        if (team.is_master() && il[k] < cnt) {  // master-only epilogue
          const int64_t n = n0 + il[k];
          out[n] = init ? Op::apply(init[n], res) : res;
        }
      }
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[st]);  // this warp is done with the stage
  }
}

// ---------------------------------------------------------------- host side
static constexpr size_t kRtSmemPerCTA = 227 * 1024;

// Launch shape: stages of ~stage_bytes (default 64 KB: measured on C3,
// profiles/reduce_tma_explore_r01g.jsonl -- 64 KB stages beat 32 KB by 10-40 %
// and 16 KB by 1.5-2x), as many as fit one CTA per SM (<= 6), persistent grid
// of one CTA per SM.
template <class T, class Op, int S, int DIST>
static int launch_reduce_tma(const void* in, const void* init, void* out, int64_t N, int64_t L,
                             int stage_bytes, int stages, cudaStream_t st, LaunchInfo* info) {
  const int64_t item_bytes = L * (int64_t)sizeof(T);
  const int64_t target = stage_bytes > 0 ? stage_bytes : 65536;
  int64_t ips = target / item_bytes;
  if (ips < 1) ips = 1;
  if (ips > N && N > 0) ips = N;
  const int64_t tile = ips * item_bytes;
  int nst = stages > 0 ? stages : (int)((kRtSmemPerCTA - rt_header_bytes(8)) / tile);
  if (stages <= 0 && nst > 6) nst = 6;
  const size_t smem = rt_header_bytes(nst) + (size_t)nst * tile;
  if (nst < 2 || smem > kRtSmemPerCTA) {
    set_error("TMA-staged reduce: a ring of >= 2 stages of %lld B does not fit 227 KB", (long long)tile);
    return CUDANP_ERR_UNSUPPORTED;
  }
  auto kern = reduce_tma_kernel<T, Op, S, DIST>;
  const int64_t nchunks = (N + ips - 1) / ips;
  const int64_t grid = nchunks < sm_count() ? nchunks : sm_count();
  if (info) {
    info->block_threads = kRtThreads;
    info->grid = grid;
    info->smem = (int)smem;
    info->map = MAP_INTRA;
    kernel_attrs(kern, &info->regs, nullptr);
    return CUDANP_OK;
  }
  if (N == 0) return CUDANP_OK;
  if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return check_launch("reduce_tma smem attribute");
  launch_pdl(kern, dim3((unsigned)grid), dim3(kRtThreads), smem, st, (const T*)in, (const T*)init,
             (T*)out, N, L, (int)ips, nst);
  return check_launch("reduce_tma launch");
}

template <class T, class Op>
static int reduce_tma_t(const void* in, const void* init, void* out, int64_t N, int64_t L, int S,
                        int dist, int stage_bytes, int stages, cudaStream_t st, LaunchInfo* info) {
  CUDANP_DISPATCH_S(S, {
    return dist == DIST_CYCLIC
               ? launch_reduce_tma<T, Op, kS, DIST_CYCLIC>(in, init, out, N, L, stage_bytes, stages, st, info)
               : launch_reduce_tma<T, Op, kS, DIST_BLOCK>(in, init, out, N, L, stage_bytes, stages, st, info);
  });
  return CUDANP_OK;
}

// Preconditions (checked by the ABI): `in` 16-byte aligned, L % 4 == 0, L > 0.
int reduce_tma(const void* in, const void* init, void* out, int64_t N, int64_t L, int dtype, int op,
               int S, int dist, int stage_bytes, int stages, cudaStream_t st, LaunchInfo* info) {
  if (dtype == CUDANP_F32)
    return op == CUDANP_SUM
               ? reduce_tma_t<float, OpSum>(in, init, out, N, L, S, dist, stage_bytes, stages, st, info)
               : reduce_tma_t<float, OpMax>(in, init, out, N, L, S, dist, stage_bytes, stages, st, info);
  return op == CUDANP_SUM
             ? reduce_tma_t<int32_t, OpSum>(in, init, out, N, L, S, dist, stage_bytes, stages, st, info)
             : reduce_tma_t<int32_t, OpMax>(in, init, out, N, L, S, dist, stage_bytes, stages, st, info);
}

}  // namespace cudanp
