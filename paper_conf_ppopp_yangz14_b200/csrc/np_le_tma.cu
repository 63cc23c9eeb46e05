// np_le_tma.cu -- the LE multi-section item (Figs 5-6) with
// the live array Grad in SHARED memory (Fig 6b), filled by TMA.
//
// Fig 6 offers three homes for the local array Grad[NPOINTS] once its loops
// are shared by a team: a global array (6a), a shared-memory array indexed by
// the master (6b), or a partition into per-slave register arrays (6c); Fig 15
// measures all three.  np_le.cu holds 6c (the default) and the
// re-read-the-input form of 6a; this file is 6b, B200-style: items are
// contiguous in the item-major layout, so a run of `ips` consecutive items is
// one block of ips*L*4 bytes that a producer warp streams into a ring of
// shared-memory stages with 1-D bulk copies (cp.async.bulk + mbarrier).  The
// stage IS the Grad array of its ips masters: the S-lane teams (intra-warp,
// P:189-191) run loop 1+2 over their share (cyclic P:166 / block R5), reduce
// the sum, every lane forms ave = sum / L (uniform), loop 3
// re-reads the share from shared memory, var and ep are reduced
// and the master stores.  Each slave visits its elements in the
// same order as the register version, so results are bit-identical to it.
#include "common.cuh"
#include "np_le_acc.cuh"
#include "np_team.cuh"
#include "np_tma.cuh"

namespace cudanp {

#ifndef CUDANP_LT_WARPS
#define CUDANP_LT_WARPS 16
#endif
constexpr int kLtWarps = CUDANP_LT_WARPS;         // consumer warps per CTA
constexpr int kLtThreads = 32 * (kLtWarps + 1);   // + one producer warp

static __host__ __device__ __forceinline__ size_t lt_header_bytes(int stages) {
  return 128 * ((16 * (size_t)stages + 127) / 128);
}

template <int S, int DIST>
__global__ void __launch_bounds__(kLtThreads, 1)
le_tma_kernel(const float* __restrict__ in, float* gicov, float* ave_out, float* var_out,
              float* ep_out, int64_t N, int64_t L, float thr, int ips, int stages) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw);
  uint64_t* empty = full + stages;
  float* ring = reinterpret_cast<float*>(smem_raw + lt_header_bytes(stages));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t nchunks = (N + ips - 1) / ips;
  const int64_t stage_elems = (int64_t)ips * L;
  const int64_t mine = (int64_t)blockIdx.x < nchunks ? (nchunks - 1 - blockIdx.x) / gridDim.x + 1 : 0;

  if (threadIdx.x == 0) {
    for (int i = 0; i < stages; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], kLtWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  if (warp == kLtWarps) {  // producer: loop 1's reads, as bulk copies of whole items
    if (lane == 0) {
      for (int64_t t = 0; t < mine; ++t) {
        const int st = (int)(t % stages);
        if (t >= stages) mbar_wait(&empty[st], (uint32_t)((t / stages) - 1) & 1);
        const int64_t n0 = ((int64_t)blockIdx.x + t * gridDim.x) * ips;
        const int64_t cnt = N - n0 < ips ? N - n0 : ips;
        const uint32_t bytes = (uint32_t)(cnt * L * 4);
        mbar_expect_tx(&full[st], bytes);
        bulk_load_1d(ring + st * stage_elems, in + n0 * L, bytes, &full[st]);
      }
    }
    return;
  }

  constexpr int TPW = 32 / S;
  constexpr int HM = (3 + S - 1) / S;
  const IntraTeam<S> team;
  const int sl = team.slave;
  for (int64_t t = 0; t < mine; ++t) {
    const int st = (int)(t % stages);
    const int64_t n0 = ((int64_t)blockIdx.x + t * gridDim.x) * ips;
    const int cnt = (int)(N - n0 < ips ? N - n0 : ips);
    mbar_wait(&full[st], (uint32_t)(t / stages) & 1);
    const float* base = ring + st * stage_elems;
    const int ntile = (cnt + TPW - 1) / TPW;
    for (int tile = warp; tile < ntile; tile += kLtWarps) {
      const int il = tile * TPW + team.team;
      const bool ok = il < cnt;
      const float* Grad = base + (int64_t)(ok ? il : 0) * L;  // DEF_Grad (Fig 6b)
      // The register version's element order (np_le.cu LeSlaveV): head up to
      // the row's 16-byte boundary (global and shared offsets agree: every
      // run starts 16-byte aligned), 128-bit body units, tail.
      const int64_t Lr = ok ? L : 0;
      int64_t hh = (4 - (int64_t)(((uintptr_t)(in + (n0 + il) * L) >> 2) & 3)) & 3;
      if (hh > Lr) hh = Lr;
      const int64_t nu = (Lr - hh) >> 2;
      const int h = (int)hh, tl = (int)(Lr - hh - 4 * nu);
      const Range<S, DIST> r(nu, 4 * nu, 4, sl);  // body units of this slave (P:166 / R5)
      const float* body = Grad + hh;
      const float* trow = body + 4 * nu;
      auto unit = [&](int64_t u) {
        const float4 v = *reinterpret_cast<const float4*>(body + 4 * u);
        return V4<float>{v.x, v.y, v.z, v.w};
      };
      LeSum acc;                                                      // loops 1+2
#pragma unroll
      for (int j = 0; j < HM; ++j) acc.head(sl + j * S < h ? Grad[sl + j * S] : 0.f);
      for (int64_t u = r.begin; u < r.end; u += r.step) acc.body(unit(u));
#pragma unroll
      for (int j = 0; j < HM; ++j) acc.tail(sl + j * S < tl ? trow[sl + j * S] : 0.f);
      const float sum = team.template reduce<OpSum>(acc.result());
      const float ave = sum / (float)L;
      LeVarEp a(ave);                                                 // loop 3
#pragma unroll
      for (int j = 0; j < HM; ++j)
        if (sl + j * S < h) a.head(Grad[sl + j * S]);
      for (int64_t u = r.begin; u < r.end; u += r.step) a.body(unit(u));
#pragma unroll
      for (int j = 0; j < HM; ++j)
        if (sl + j * S < tl) a.tail(trow[sl + j * S]);
      float var = a.var(), ep = a.ep();
      var = team.template reduce<OpSum>(var);
      ep = team.template reduce<OpSum>(ep);
      if (team.is_master() && ok) {
        const int64_t n = n0 + il;
        if ((ave * ave) / var > thr) gicov[n] = ave / sqrtf(var);
        if (ave_out) ave_out[n] = ave;
        if (var_out) var_out[n] = var;
        if (ep_out) ep_out[n] = ep;
      }
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[st]);
  }
}

// ---------------------------------------------------------------- point-major (layout 1)
// The same placement for point-major data in[i*N + n], the inter-warp map
// (the paper's choice for LE): 32 adjacent items are the masters (one
// per lane) and S slave warps share the points.  A group's Grad array is the
// box [32 items x L points] -- 128 bytes per point, coalesced -- that a
// producer warp streams into the ring with one 2-D TMA copy; slave s runs
// loops 1+2 over its points (cyclic P:166 / block R5) reading
// ring[point][lane], the S partial sums meet in shared memory and
// every slave folds them (in slave order) into ave itself -- a uniform value
// recomputed rather than broadcast, which saves a barrier; loop 3
// re-reads the points from shared memory and var / ep are folded by the
// master before it stores.  The
// producer runs up to `stages` groups ahead, so the next groups' bytes are
// in flight while the slaves reduce (the register version idles its loads
// during each group's reductions and barriers).  The slaves sync among
// themselves with a named barrier (the producer warp never waits on it).
// Each slave pairs its iterations exactly as LeSlave does (np_le.cu), so the
// results are bit-identical to the register placement.
template <int S, int DIST>
__global__ void __launch_bounds__(32 * (S + 1), 1)
le_tma_pm_kernel(const __grid_constant__ CUtensorMap map, float* gicov, float* ave_out,
                 float* var_out, float* ep_out, int64_t N, int64_t L, float thr, int stages) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  __shared__ float red[2][S][33], red2[2][S][33];  // double-buffered by group parity
  uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw);
  uint64_t* empty = full + stages;
  float* ring = reinterpret_cast<float*>(smem_raw + lt_header_bytes(stages));  // [stages][L][32]
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t ngroups = (N + 31) / 32;
  const int64_t mine = (int64_t)blockIdx.x < ngroups ? (ngroups - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  const int64_t stage_elems = L * 32;
  if (threadIdx.x == 0) {
    for (int i = 0; i < stages; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], S);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == S) {  // producer: loop 1's reads, one box per group of 32 masters
    if (lane == 0) {
      for (int64_t t = 0; t < mine; ++t) {
        const int st = (int)(t % stages);
        if (t >= stages) mbar_wait(&empty[st], (uint32_t)((t / stages) - 1) & 1);
        const int64_t g = blockIdx.x + t * gridDim.x;
        mbar_expect_tx(&full[st], (uint32_t)(stage_elems * 4));
        tma_load_2d(ring + st * stage_elems, &map, (int)(g * 32), 0, &full[st]);
      }
    }
    return;
  }
  auto team_sync = [] { asm volatile("bar.sync 1, %0;" ::"n"(32 * S) : "memory"); };
  const Range<S, DIST> r(L, L, 1, warp);  // this slave's points
  const int cnt = r.end > r.begin ? (int)((r.end - r.begin + r.step - 1) / r.step) : 0;
  const int64_t pstep = r.step * 32;
  for (int64_t t = 0; t < mine; ++t) {
    const int st = (int)(t % stages), par = (int)(t & 1);
    const int64_t n = (blockIdx.x + t * gridDim.x) * 32 + lane;
    const bool ok = n < N;
    mbar_wait(&full[st], (uint32_t)(t / stages) & 1);
    const float* p0 = ring + st * stage_elems + r.begin * 32 + lane;  // DEF_Grad (Fig 6b)
    // loops 1+2, consecutive iterations in pairs (FADD2), as LeSlave::loop12
    float2 s2 = make_float2(0.f, 0.f);
    int c = 0;
    for (; c + 1 < cnt; c += 2) s2 = __fadd2_rn(s2, make_float2(p0[c * pstep], p0[(c + 1) * pstep]));
    if (c < cnt) s2.x += p0[c * pstep];
    red[par][warp][lane] = s2.x + s2.y;
    team_sync();
    float sm = red[par][0][lane];  // sum = reduction(sum) in slave order
#pragma unroll
    for (int k = 1; k < S; ++k) sm += red[par][k][lane];
    const float ave = sm / (float)L;  // P:309, recomputed by every slave
    // loop 3, pairs as LeSlave::loop3
    const float2 na = make_float2(-ave, -ave);
    float2 v2 = make_float2(0.f, 0.f), e2 = make_float2(0.f, 0.f);
    for (c = 0; c < cnt; c += 2) {
      const bool vb = c + 1 < cnt;
      float2 tt = __fadd2_rn(make_float2(p0[c * pstep], vb ? p0[(c + 1) * pstep] : 0.f), na);
      tt.y = vb ? tt.y : 0.f;
      v2 = __ffma2_rn(tt, tt, v2);
      e2 = __fadd2_rn(e2, tt);
    }
    red[par][warp][lane] = v2.x + v2.y;
    red2[par][warp][lane] = e2.x + e2.y;
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[st]);  // this slave is done with the group's Grad
    team_sync();
    if (warp == 0 && ok) {  // var, ep = reduction(.); the master stores
      float v = red[par][0][lane], pp = red2[par][0][lane];
      for (int k = 1; k < S; ++k) { v += red[par][k][lane]; pp += red2[par][k][lane]; }
      if ((ave * ave) / v > thr) gicov[n] = ave / sqrtf(v);
      if (ave_out) ave_out[n] = ave;
      if (var_out) var_out[n] = v;
      if (ep_out) ep_out[n] = pp;
    }
  }
}

// ---------------------------------------------------------------- host side
static constexpr size_t kLtSmemPerCTA = 227 * 1024;

template <int S, int DIST>
static int launch_le_tma(const float* in, float* g, float* a, float* v, float* p, int64_t N,
                         int64_t L, float thr, cudaStream_t st) {
  // ips: ~64 KB stages, a multiple of 4/gcd(L,4) items so every run starts
  // 16-byte aligned and spans a multiple of 16 bytes.
  const int64_t q = (L % 4 == 0) ? 1 : (L % 2 == 0 ? 2 : 4);
  int64_t ips = (65536 / (L * 4)) / q * q;
  if (ips < q) ips = q;
  const int64_t tile = ips * L * 4;
  int nst = (int)((kLtSmemPerCTA - lt_header_bytes(8)) / tile);
  if (nst > 6) nst = 6;
  if (nst < 2) {
    set_error("shared-memory Grad: an item of %lld B leaves no room for a 2-stage ring", (long long)(L * 4));
    return CUDANP_ERR_UNSUPPORTED;
  }
  const size_t smem = lt_header_bytes(nst) + (size_t)nst * tile;
  auto kern = le_tma_kernel<S, DIST>;
  const int64_t nchunks = (N + ips - 1) / ips;
  const int64_t grid = nchunks < sm_count() ? nchunks : sm_count();
  if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return check_launch("le_tma smem attribute");
  kern<<<(unsigned)grid, kLtThreads, smem, st>>>(in, g, a, v, p, N, L, thr, (int)ips, nst);
  return check_launch("le_gicov (shared-memory Grad) launch");
}

int le_np(const float*, float*, float*, float*, float*, int64_t, int64_t, float, int, int, int, int,
          bool, cudaStream_t);

typedef CUresult (*EncodeTiledFnLe)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                    const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                    const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                    CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

template <int S, int DIST>
static int launch_le_tma_pm(const float* in, float* g, float* a, float* v, float* p, int64_t N,
                            int64_t L, float thr, cudaStream_t st) {
  static EncodeTiledFnLe enc = nullptr;
  if (!enc) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) != cudaSuccess || !f) {
      cudaGetLastError();
      set_error("cuTensorMapEncodeTiled entry point unavailable");
      return CUDANP_ERR_CUDA;
    }
    enc = (EncodeTiledFnLe)f;
  }
  CUtensorMap map;
  const cuuint64_t dims[2] = {(cuuint64_t)N, (cuuint64_t)L};
  const cuuint64_t strides[1] = {(cuuint64_t)N * 4};
  const cuuint32_t box[2] = {32, (cuuint32_t)L};
  const cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(in), dims, strides, box,
                   estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    set_error("cuTensorMapEncodeTiled failed (%d)", (int)r);
    return CUDANP_ERR_CUDA;
  }
  // three CTAs per SM (the slaves' reductions and barriers need the extra
  // warps; ncu saw one 9-warp CTA per SM consumer-bound), each with as many
  // group stages as a third of the SM's shared memory holds (<= 8)
  const size_t stage = (size_t)L * 32 * 4;
  int nst = (int)((72 * 1024 - lt_header_bytes(8)) / stage);
  if (nst > 8) nst = 8;
  if (nst < 2) {
    set_error("shared-memory Grad (point-major): %lld points leave no room for a 2-stage ring", (long long)L);
    return CUDANP_ERR_UNSUPPORTED;
  }
  const size_t smem = lt_header_bytes(nst) + (size_t)nst * stage;
  auto kern = le_tma_pm_kernel<S, DIST>;
  if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess ||
      cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100) != cudaSuccess)
    return check_launch("le_tma (point-major) smem attributes");
  const int64_t grid = persistent_grid(kern, 32 * (S + 1), smem, (N + 31) / 32);
  kern<<<(unsigned)grid, 32 * (S + 1), smem, st>>>(map, g, a, v, p, N, L, thr, nst);
  return check_launch("le_gicov (shared-memory Grad, point-major) launch");
}

// Point-major shared-memory Grad: inter-warp, S <= 16 (a producer warp beside
// S slave warps) incl. 3, 5, 10, 15; needs N % 4 == 0 (row pitch), L <= 256
// (one TMA box per group) and a 16-byte aligned input (the ABI checks).
int le_tma_pm(const float* in, float* gicov, float* ave, float* var, float* ep, int64_t N, int64_t L,
              float thr, int S, int dist, cudaStream_t st) {
  if (N == 0) return CUDANP_OK;
#define CUDANP_LE_PM(KS)                                                                             \
  case KS:                                                                                           \
    return dist == DIST_CYCLIC ? launch_le_tma_pm<KS, DIST_CYCLIC>(in, gicov, ave, var, ep, N, L, thr, st) \
                               : launch_le_tma_pm<KS, DIST_BLOCK>(in, gicov, ave, var, ep, N, L, thr, st);
  switch (S) {
    CUDANP_LE_PM(1) CUDANP_LE_PM(2) CUDANP_LE_PM(3) CUDANP_LE_PM(4) CUDANP_LE_PM(5)
    CUDANP_LE_PM(8) CUDANP_LE_PM(10) CUDANP_LE_PM(15) CUDANP_LE_PM(16)
    default:
      set_error("shared-memory Grad (point-major) is built for S in {1,2,3,4,5,8,10,15,16}");
      return CUDANP_ERR_UNSUPPORTED;
  }
#undef CUDANP_LE_PM
}

// Preconditions (checked by the ABI): item-major, in 16-byte aligned,
// intra-warp map, S a power of two <= 32.  Bulk copies move multiples of 16
// bytes, so the ring takes the first N_main items (a multiple of 4/gcd(L,4))
// and the < 4 last items go through the register-partition kernel -- same
// per-slave order, same results.
int le_tma(const float* in, float* gicov, float* ave, float* var, float* ep, int64_t N, int64_t L,
           float thr, int S, int dist, cudaStream_t st) {
  if (N == 0) return CUDANP_OK;
  const int64_t q = (L % 4 == 0) ? 1 : (L % 2 == 0 ? 2 : 4);
  const int64_t Nm = N / q * q;
  if (Nm > 0) {
    int rc = CUDANP_OK;
    CUDANP_DISPATCH_S(S, {
      rc = dist == DIST_CYCLIC ? launch_le_tma<kS, DIST_CYCLIC>(in, gicov, ave, var, ep, Nm, L, thr, st)
                               : launch_le_tma<kS, DIST_BLOCK>(in, gicov, ave, var, ep, Nm, L, thr, st);
    });
    if (rc) return rc;
  }
  if (Nm == N) return CUDANP_OK;
  auto off = [&](float* p) { return p ? p + Nm : nullptr; };
  return le_np(in + Nm * L, gicov + Nm, off(ave), off(var), off(ep), N - Nm, L, thr, 0, S, dist,
               MAP_INTRA, false, st);
}

}  // namespace cudanp
