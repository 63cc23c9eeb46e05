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
