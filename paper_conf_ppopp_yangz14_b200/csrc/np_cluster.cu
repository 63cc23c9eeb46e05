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

template <class T, class Op>
__device__ __forceinline__ V4<T> cop4(V4<T> a, V4<T> b) {
  return {Op::apply(a.x, b.x), Op::apply(a.y, b.y), Op::apply(a.z, b.z), Op::apply(a.w, b.w)};
}

template <class T, class Op, int S, int DIST, bool VEC>
__global__ void __launch_bounds__(S / kClusterCtas)
reduce_cluster_kernel(const T* __restrict__ in, const T* __restrict__ init, T* __restrict__ out,
                      int64_t N, int64_t L) {
  pdl_entry();
  constexpr int CTA = S / kClusterCtas;
  constexpr int W = CTA / 32;
  __shared__ T wsum[W];
  __shared__ T part[2][kClusterCtas];  // the master CTA's receive slots, double-buffered
  cg::cluster_group cluster = cg::this_cluster();
  const int rank = (int)cluster.block_rank();
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int slave = rank * CTA + tid;  // slave id within the cluster-wide team
  const int64_t nunits = VEC ? (L >> 2) : L;
  const Range<S, DIST> r(nunits, L, VEC ? 4 : 1, slave);
  const int64_t cid = blockIdx.x / kClusterCtas, ncl = gridDim.x / kClusterCtas;
  const T id = Op::template identity<T>();
  T* master_part = cluster.map_shared_rank(&part[0][0], 0);
  // A CTA may touch another CTA's shared memory only once that CTA is known
  // to be running: arrive on the cluster barrier now, wait for it just before
  // the first DSMEM store (the first item's loads overlap the wait).
  asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
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
    // Team reduction, level 1: shfl inside each warp ...
    T p = Op::apply(Op::apply(acc.x, acc.y), Op::apply(acc.z, acc.w));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) p = Op::apply(p, __shfl_xor_sync(kFull, p, o));
    // ... level 2: the CTA's warps through shared memory ...
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
      // ... level 3: the CTA's partial into the master CTA's slot over DSMEM.
      master_part[par * kClusterCtas + rank] = c;
    }
    cluster.sync();  // release/acquire: every slot is visible to rank 0; wsum reusable
    if (rank == 0 && tid == 0) {  // the master finishes the item alone
      T res = part[par][0];
#pragma unroll
      for (int k = 1; k < kClusterCtas; ++k) res = Op::apply(res, part[par][k]);
      out[item] = init ? Op::apply(init[item], res) : res;
    }
    // Slots [par] are rewritten two items later, after the next cluster.sync,
    // which rank 0 reaches only after reading them.
  }
  if (!started) asm volatile("barrier.cluster.wait.aligned;" ::: "memory");
}

#define CUDANP_DISPATCH_CLUSTER_S(S, ...)                      \
  switch (S) {                                                 \
    case 2048: { constexpr int kS = 2048; __VA_ARGS__; } break; \
    case 4096: { constexpr int kS = 4096; __VA_ARGS__; } break; \
    case 8192: { constexpr int kS = 8192; __VA_ARGS__; } break; \
    default: return fail_invalid("S must be 2048, 4096 or 8192 for a cluster team"); \
  }

template <class T>
static int launch_cluster(void (*kern)(const T*, const T*, T*, int64_t, int64_t), int cta, int64_t N,
                          cudaStream_t st, LaunchInfo* info, const T* in, const T* init, T* out,
                          int64_t L) {
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
    cudaGetLastError();
    resident = 1;
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
  cudaError_t e = cudaLaunchKernelEx(&cfg, kern, in, init, out, N, L);
  if (e != cudaSuccess) {
    set_error("batched_loop_reduce (cluster team) launch: %s", cudaGetErrorString(e));
    cudaGetLastError();
    return CUDANP_ERR_CUDA;
  }
  return check_launch("batched_loop_reduce (cluster team) launch");
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
    return launch_cluster<T>(kern, CTA, N, st, info, (const T*)in, (const T*)init, (T*)out, L);
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

}  // namespace cudanp
