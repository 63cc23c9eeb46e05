// abi.cu -- the extern "C" boundary of libcudanp.so (include/cudanp.h):
// argument validation before any launch, choice of map / vector path,
// dispatch to the kernels, status codes and error text.  Also the device-side
// input generator and the debug exports that run the kernels' own team and
// distribution code.
#include <cstdarg>
#include <cstdlib>

#include "common.cuh"
#include "np_team.cuh"

namespace cudanp {

// ---- kernels' host entry points (np_reduce.cu, np_scan.cu, np_matvec.cu, np_dp.cu)
int reduce_np(const void*, const void*, void*, int64_t, int64_t, int, int, int, int, int, bool,
              cudaStream_t, LaunchInfo*);
int reduce_literal(const void*, const void*, void*, int64_t, int64_t, int, int, cudaStream_t);
int reduce_backend(const void*, const void*, void*, int64_t, int64_t, int, int, int, int,
                   cudaStream_t);
int scan_np(const void*, const void*, void*, int64_t, int64_t, int, int, int, int, bool,
            cudaStream_t, LaunchInfo*);
int scan_literal(const void*, const void*, void*, int64_t, int64_t, int, cudaStream_t);
int tmv_np(const float*, int64_t, const float*, float*, int64_t, int64_t, int, int, int, bool,
           cudaStream_t, LaunchInfo*);
int mv_np(const float*, int64_t, const float*, float*, int64_t, int64_t, int, int, int, bool,
          cudaStream_t, LaunchInfo*);
int tmv_literal(const float*, int64_t, const float*, float*, int64_t, int64_t, cudaStream_t);
int mv_literal(const float*, int64_t, const float*, float*, int64_t, int64_t, cudaStream_t);
int dp_tmv(bool, const float*, int64_t, const float*, float*, int64_t, int64_t, cudaStream_t);
int dp_mv(bool, const float*, int64_t, const float*, float*, int64_t, int64_t, cudaStream_t);
int dp_reduce(bool, const void*, const void*, void*, int64_t, int64_t, int, int, cudaStream_t);
int dp_scan(bool, const void*, const void*, void*, int64_t, int64_t, int, cudaStream_t);
int dp_error_count(int, int64_t*);
int dp_memcopy(const float*, float*, int64_t, int64_t, int, cudaStream_t);
int tmv_tma(const float*, int64_t, const float*, float*, int64_t, int64_t, int, int, int, int, int,
            cudaStream_t, LaunchInfo*);
int reduce_tma(const void*, const void*, void*, int64_t, int64_t, int, int, int, int, int, int,
               cudaStream_t, LaunchInfo*);
int ragged_np(const void*, const int64_t*, const void*, void*, int64_t, int, int, int, int, int,
              cudaStream_t);
int ragged_literal(const void*, const int64_t*, const void*, void*, int64_t, int, int, cudaStream_t);
int ragged_adaptive(const void*, const int64_t*, const void*, void*, int64_t, int, int, int64_t,
                    cudaStream_t);
int le_np(const float*, float*, float*, float*, float*, int64_t, int64_t, float, int, int, int, int,
          bool, cudaStream_t);
int le_tma(const float*, float*, float*, float*, float*, int64_t, int64_t, float, int, int,
           cudaStream_t);
int mv_s1_tiled(const float*, int64_t, const float*, float*, int64_t, int64_t, cudaStream_t);
int scan_s1_tiled(const void*, const void*, void*, int64_t, int64_t, int, cudaStream_t);
int reduce_s1_tiled(const void*, const void*, void*, int64_t, int64_t, int, int, cudaStream_t);
int le_tma_pm(const float*, float*, float*, float*, float*, int64_t, int64_t, float, int, int,
              cudaStream_t);
int le_literal(const float*, float*, float*, float*, float*, int64_t, int64_t, float, int,
               cudaStream_t);

static thread_local char g_err[512] = "";

void set_error(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
}

int sm_count() {
  static int cache[64] = {0};
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return 148; }
  if (dev < 0 || dev >= 64) dev = 0;
  if (!cache[dev]) {
    int n = 0;
    if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n < 1) {
      cudaGetLastError();
      n = 148;
    }
    cache[dev] = n;
  }
  return cache[dev];
}

bool pdl_enabled() {
  static const bool on = [] {
    const char* e = getenv("CUDANP_PDL");
    return !(e && e[0] == '0');
  }();
  return on;
}

// ---------------------------------------------------------------- validation
static bool size_ok(int64_t a, int64_t b) {  // a*b*4 bytes addressable
  if (a < 0 || b < 0) return false;
  if (a == 0 || b == 0) return true;
  return a <= (INT64_MAX / 8) / b;
}

// inter_ok: the call also builds the non-power-of-two inter-warp teams
// (valid_inter_S; intra-warp then returns CUDANP_ERR_UNSUPPORTED).
static int check_common(int S, int dist, int map, int64_t n_outer, int64_t n_inner,
                        bool cluster_ok = false, bool inter_ok = false) {
  if (!valid_S(S) && !valid_big_S(S) && !(cluster_ok && valid_cluster_S(S)) &&
      !(inter_ok && valid_inter_S(S)))
    return fail_invalid(cluster_ok ? "S must be one of 1,2,4,8,16,32 (3,5,10,15 inter-warp; 64..1024 "
                                     "multi-warp teams, 2048/4096/8192 cluster teams)"
                                   : "S must be one of 1,2,4,8,16,32 (3,5,10,15 inter-warp; 64..1024 "
                                     "multi-warp teams)");
  if (dist != CUDANP_DIST_CYCLIC && dist != CUDANP_DIST_BLOCK) return fail_invalid("dist");
  if (map != CUDANP_MAP_AUTO && map != CUDANP_MAP_INTRA_WARP && map != CUDANP_MAP_INTER_WARP)
    return fail_invalid("map");
  if (valid_inter_S(S) && map == CUDANP_MAP_INTRA_WARP) {
    set_error("intra-warp teams need S = 2^k <= 32 (P:342); S = %d runs with the inter-warp map "
              "(P:447)", S);
    return CUDANP_ERR_UNSUPPORTED;
  }
  if (n_outer < 0 || n_inner < 0) return fail_invalid("negative size");
  if (!size_ok(n_outer, n_inner)) return fail_invalid("size overflows int64 byte offsets");
  return CUDANP_OK;
}

static int check_dtype_op(int dtype, int op) {
  if (dtype != CUDANP_F32 && dtype != CUDANP_I32) return fail_invalid("dtype");
  if (op != CUDANP_SUM && op != CUDANP_MAX) return fail_invalid("op");
  return CUDANP_OK;
}

// MAP_AUTO per P:340-342 / P:486: keep the access pattern coalesced.  TMV's
// masters (columns) are adjacent in memory -> inter-warp; MV rows and
// item-major reduce/scan rows are contiguous per master -> intra-warp.
// A team that is not a power of two exists only as an inter-warp team.
static int resolve_map(int map, bool is_tmv, int S = 1) {
  if (map != CUDANP_MAP_AUTO) return map;
  return (is_tmv || valid_inter_S(S)) ? MAP_INTER : MAP_INTRA;
}

// ---------------------------------------------------------------- version choice
static int floor_pow2(int64_t v) {
  int p = 1;
  while ((int64_t)p * 2 <= v && p < (1 << 30)) p *= 2;
  return p;
}
static int clampi(int v, int lo, int hi) { return v < lo ? lo : (v > hi ? hi : v); }

// TMA staging of TMV pays while the 128-column strips give between ~0.3 and
// ~1.1 CTAs per SM: one resident strip per SM with a deep ring of 32-64 KB
// stages (profiles/tmv_width_r02d.jsonl: w = 8192..20480 at h = 16384/65536,
// TMA 6.3-7.2 TB/s vs LDG 6.0-7.2).  Narrower (C1, 1024 columns: TMA S = 32
// 5.1 us vs LDG inter-warp 3.2 us, profiles/sweep_r01n.jsonl; w = 4096: 4.1 vs
// 4.7 TB/s) the LDG kernel with more slaves per column spreads the few
// columns better; wider (w >= 24576: several strips per SM, smaller stages)
// the LDG inter-warp kernel with S = 32 holds 6.8-7.3 TB/s where the TMA
// ring's shape swings from 4.1 to 7.2.
static bool tmv_wide(int64_t w) {
  const int64_t strips = (w + 127) / 128, sms = sm_count();
  return 10 * strips >= 3 * sms && 10 * strips <= 11 * sms;
}
// TMA preconditions: A 16-byte aligned, row pitch a multiple of 16 bytes,
// coordinates in int32, something to stream.  y is stored with scalar stores
// and x with ordinary loads, so neither needs alignment.
static bool tma_ok(const float* A, int64_t lda, int64_t w, int64_t h) {
  return aligned16(A) && lda % 4 == 0 && w > 0 && h > 0 && w < (int64_t(1) << 31) &&
         h < (int64_t(1) << 31);
}

// The library's choice of (S, dist, map) when the caller passes S = 0
// (CUDANP_S_AUTO): the paper picks the version by exhaustive search (P:413,
// P:486); this rule encodes what that search found on B200 (DESIGN.md §6,
// profiles/sweep_r01n.jsonl, bench_r01*.json), so no call has to time
// anything.  T = SMs x 1024 threads is "enough threads to fill the GPU":
// when N x S falls short, the team grows (NP pays when outer
// TLP is short), up to a team whose slaves still get >= 8 elements each.
//   TMV: tmv_wide + TMA-able -> TMA, S = 8 cyclic (C2 best), except below
//        0.75 strips per SM on aligned matrices (-> the S = 128 rule below);
//        wider than that -> LDG inter-warp S = 32 block; narrower -> LDG inter-warp with
//        S = 128 when 16-byte aligned (else clamp(2T / w, 8, 64)), block when
//        each slave's share is < 32 rows and w > 1024, cyclic otherwise (C1:
//        128 cyclic; profiles/tmv_narrow_new_r02a[ef].jsonl: S = 128 best for
//        w <= 4096 at every h but w = 512).
//   MV:  intra, S = clamp(L / 64, 1, 256) cyclic (C2 best: S = 256), grown.
//   reduce: intra, S = clamp(L / 8, 1, 32) (C3: 4/8/16/32 at L = 32..256),
//        block above L = 32 (L % 4 != 0: L / 16), grown.
//   scan: intra, S = clamp(L / 4, 1, 16) (C4: 16), cyclic from L = 128, grown.
// A map other than AUTO is kept (and the S chosen for it).
int choose_version(int op_kind, int64_t N, int64_t L, bool vec, bool tma, int map_in, int* S,
                   int* dist, int* map) {
  const int64_t T = (int64_t)sm_count() * 1024;
  auto grow = [&](int s, int cap) {
    while ((int64_t)s * 2 <= cap && N * s < T) s *= 2;
    return s;
  };
  const int cap_l8 = clampi(floor_pow2(L / 8), 1, 1024);
  int s = 1, d = CUDANP_DIST_CYCLIC, m = map_in;
  switch (op_kind) {
    case 0: {  // TMV: N = w columns, L = h rows
      // the lower part of the TMA band goes to the 128-bit S = 128 LDG team
      // when the matrix is aligned (width sweep r02ak: w = 8192 / 12288
      // 6987 / 6790 vs 6272 / 6617 GB/s for the best TMA version)
      const bool lower = vec && 4 * ((N + 127) / 128) < 3 * (int64_t)sm_count();
      if (tma && tmv_wide(N) &&
          (map_in == CUDANP_MAP_INTER_WARP_TMA || (map_in == CUDANP_MAP_AUTO && !lower))) {
        s = 8; d = CUDANP_DIST_CYCLIC; m = CUDANP_MAP_INTER_WARP_TMA;
        break;
      }
      if (m == CUDANP_MAP_INTER_WARP_TMA) m = CUDANP_MAP_INTER_WARP;  // fallback (not TMA-able)
      if (m == CUDANP_MAP_INTRA_WARP) {
        s = clampi(floor_pow2(N > 0 ? T / N : 32), 1, 32);
      } else if (10 * ((N + 127) / 128) > 11 * (int64_t)sm_count()) {
        m = CUDANP_MAP_INTER_WARP;  // wide: several strips per SM
        s = 32;
        d = CUDANP_DIST_BLOCK;
      } else {
        m = CUDANP_MAP_INTER_WARP;  // narrow: S = 128 on aligned matrices (vec)
        s = vec ? 128 : clampi(floor_pow2(N > 0 ? 2 * T / N : 64), 8, 64);
      }
      s = clampi(s, 1, clampi(floor_pow2(L / 4), 1, 128));
      if (m == CUDANP_MAP_INTER_WARP && s != 32)
        d = L / s < 32 && (!vec || N > 1024) ? CUDANP_DIST_BLOCK : CUDANP_DIST_CYCLIC;
      break;
    }
    case 1:  // MV
      if (m == CUDANP_MAP_INTER_WARP) {
        s = clampi(floor_pow2(L / 128), 1, 32);
      } else {
        m = CUDANP_MAP_INTRA_WARP;
        s = clampi(floor_pow2(L / 64), 1, 256);
        s = grow(s, cap_l8 > s ? cap_l8 : s);
      }
      break;
    case 2:  // batched reduce
      if (m == CUDANP_MAP_INTER_WARP) {
        s = clampi(floor_pow2(L / 32), 1, 32);
      } else {
        m = CUDANP_MAP_INTRA_WARP;
        s = clampi(floor_pow2(vec ? L / 8 : L / 16), 1, 32);
        d = L > 32 ? CUDANP_DIST_BLOCK : CUDANP_DIST_CYCLIC;
        s = grow(s, cap_l8);
        if (s > 32) d = CUDANP_DIST_CYCLIC;
      }
      break;
    case 3:  // batched scan
      if (m == CUDANP_MAP_INTER_WARP) {
        s = clampi(floor_pow2(L / 32), 1, 32);
      } else {
        m = CUDANP_MAP_INTRA_WARP;
        s = clampi(floor_pow2(L / 4), 1, 16);
        d = L >= 128 ? CUDANP_DIST_CYCLIC : CUDANP_DIST_BLOCK;
        s = grow(s, cap_l8);
        if (s > 32) d = CUDANP_DIST_CYCLIC;
      }
      break;
    default:
      return fail_invalid("op_kind");
  }
  *S = s;
  *dist = d;
  *map = m;
  return CUDANP_OK;
}

static int check_tmv_args(const float* A, int64_t lda, const float* x, float* y, int64_t w,
                          int64_t h, int S, int dist, int map) {
  int rc = check_common(S, dist, map, w, h, false, true);
  if (rc) return rc;
  if (w > 0 && h > 0 && lda < w) return fail_invalid("lda < n_outer (TMV row length)");
  if (!size_ok(h, lda)) return fail_invalid("h*lda overflows");
  if (w > 0 && !y) return fail_invalid("y is NULL");
  if (w > 0 && h > 0 && (!A || !x)) return fail_invalid("A or x is NULL");
  return CUDANP_OK;
}

static int check_mv_args(const float* A, int64_t lda, const float* x, float* y, int64_t h,
                         int64_t w, int S, int dist, int map) {
  int rc = check_common(S, dist, map, h, w, true, true);
  if (rc) return rc;
  if (h > 0 && w > 0 && lda < w) return fail_invalid("lda < n_inner (MV row length)");
  if (!size_ok(h, lda)) return fail_invalid("h*lda overflows");
  if (h > 0 && !y) return fail_invalid("y is NULL");
  if (h > 0 && w > 0 && (!A || !x)) return fail_invalid("A or x is NULL");
  return CUDANP_OK;
}

// TMV masters are columns: 128-bit loads give each thread 4 adjacent
// masters (R19), which divides the CTA count by 4.  Measured on B200 (C1
// 1024^2 vs C2 16384^2, profiles/): V=4 wins as long as the 4-wide grid has at
// least half an SM's worth of CTAs per SM pair (>= SMs/2 CTAs); for narrower
// matrices one master per thread (plus 8-master CTAs, np_matvec.cu) spreads
// the few columns over more SMs.
// The CTAs of S = 64 / 128 (8 or 4 column-masters, np_matvec.cu
// launch_tmv_big) take V = 4 when its 16-column CTAs still number >= 0.8 SMs,
// or, for short columns (h <= 2048: latency-bound, one load batch per slave),
// >= a quarter of the SMs; tall narrow matrices keep V = 1's twice as many
// CTAs (bandwidth needs the SMs).  Graph of cold launches
// (profiles/tmv_narrow_*_r02ae.jsonl): h = 1024, w = 1024 / 2048 / 4096,
// S = 128: 2.39 -> 2.15, 3.33 -> 2.58, 5.55 -> 4.03 us; h = 16384, w = 1024
// stays V = 1 (19.1 vs 21.0 us).
static bool tmv_aligned(const float* A, int64_t lda, const float* y, int64_t w) {
  return (w % 4 == 0) && (lda % 4 == 0) && aligned16(A) && aligned16(y);
}
static bool tmv_vec_shape(int64_t w, int64_t h, int S) {
#if defined(CUDANP_TMV_VEC_ALWAYS)
  return true;
#else
  if (S == 64 || S == 128) {
    const int64_t ctas16 = (w + 15) / 16, sms = sm_count();
    return 10 * ctas16 >= 8 * sms || (h <= 2048 && 4 * ctas16 >= sms);
  }
  return 2 * ((w + 127) / 128) >= sm_count();
#endif
}
static bool tmv_vec(const float* A, int64_t lda, const float* y, int64_t w, int64_t h, int S) {
  return tmv_aligned(A, lda, y, w) && tmv_vec_shape(w, h, S);
}
static bool mv_vec(const float* A, int64_t lda, const float* x, int64_t w) {
  return (w % 4 == 0) && (lda % 4 == 0) && aligned16(A) && aligned16(x);
}

// ---------------------------------------------------------------- generator
// Counter-based generator, written independently of the
// oracle's copy; tests check the two agree bit for bit.
__host__ __device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__global__ void generate_kernel(void* out, int64_t rows, int64_t cols, int64_t ld, int64_t row0,
                                int64_t col0, int64_t wg, uint64_t key, int kind, int64_t B) {
  const int64_t total = rows * cols;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = e / cols, c = e - r * cols;
    const uint64_t idx = (uint64_t)(row0 + r) * (uint64_t)wg + (uint64_t)(col0 + c);
    const uint64_t h = mix64(key ^ idx);
    const int64_t o = r * ld + c;
    switch (kind) {
      case 0: ((float*)out)[o] = (float)(h >> 40 | 1ull) * 0x1p-24f; break;
      case 1: ((float*)out)[o] = (float)((int64_t)(h >> 40 | 1ull) * 2 - (1ll << 24)) * 0x1p-24f; break;
      case 2: ((float*)out)[o] = (float)(h >> 62); break;
      case 3: ((int32_t*)out)[o] = (int32_t)((int64_t)((h >> 32) & (uint64_t)(2 * B - 1)) - B); break;
      case 4: ((int32_t*)out)[o] = (int32_t)(uint32_t)(h >> 32); break;
      case 5: ((float*)out)[o] = 1.0f; break;
      case 6: ((int32_t*)out)[o] = 1; break;
      default: break;
    }
  }
}

// ---------------------------------------------------------------- memcopy (Fig 1 baseline)
// The plain copy kernel, compiled WITHOUT -rdc ("baseline ... without
// dynamic parallelism").
__global__ void memcopy_kernel(const float* __restrict__ in, float* __restrict__ out, int64_t total) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
       i += (int64_t)gridDim.x * blockDim.x)
    out[i] = in[i];
}

// ---------------------------------------------------------------- debug kernels
// Each uses the very Range / IntraTeam / InterTeam code the kernels use.
template <int S, int DIST>
__global__ void owner_kernel(int64_t L, int V, int32_t* owner) {
  const int s = threadIdx.x;
  const int64_t nunits = (L + V - 1) / V;
  const Range<S, DIST> r(nunits, L, V, s);
  for (int64_t u = r.begin; u < r.end; u += r.step)
    for (int k = 0; k < V; ++k)
      if (u * V + k < L) owner[u * V + k] = s;
}

template <int S>
__global__ void team_intra_kernel(int32_t* master, int32_t* slave) {
  const IntraTeam<S> t;
  const int tid = threadIdx.x;
  master[tid] = (tid >> 5) * IntraTeam<S>::kTeamsPerWarp + t.team;
  slave[tid] = t.slave;
}
template <int S>
__global__ void team_inter_kernel(int32_t* master, int32_t* slave) {
  const InterTeam<S> t;
  const int tid = threadIdx.y * 32 + threadIdx.x;
  master[tid] = t.master;
  slave[tid] = t.slave;
}
template <int S>
__global__ void bcast_intra_kernel(int32_t* out) {
  const IntraTeam<S> t;
  const int tid = threadIdx.x;
  out[tid] = t.read_from_master((int32_t)(1000 * tid + 7));
}
template <int S>
__global__ void bcast_inter_kernel(int32_t* out) {
  __shared__ int32_t slot[32];
  const InterTeam<S> t;
  const int tid = threadIdx.y * 32 + threadIdx.x;
  out[tid] = t.read_from_master((int32_t)(1000 * tid + 7), slot);
}

}  // namespace cudanp

using namespace cudanp;

static cudaStream_t as_stream(void* s) { return (cudaStream_t)s; }

extern "C" {

int cudanp_version(void) { return 200; }

const char* cudanp_status_string(int status) {
  switch (status) {
    case CUDANP_OK: return "CUDANP_OK";
    case CUDANP_ERR_INVALID: return "CUDANP_ERR_INVALID";
    case CUDANP_ERR_UNSUPPORTED: return "CUDANP_ERR_UNSUPPORTED";
    case CUDANP_ERR_CUDA: return "CUDANP_ERR_CUDA";
    case CUDANP_ERR_NCCL: return "CUDANP_ERR_NCCL";
    default: return "CUDANP_UNKNOWN_STATUS";
  }
}

const char* cudanp_last_error(void) { return g_err; }

// Version selection inside the call.  S = CUDANP_S_AUTO
// picks (S, dist, map) by choose_version.  MAP_AUTO takes the TMA-staged
// inter-warp kernel when its preconditions hold, S <= 32 is a power of two
// and the matrix is wide (tmv_wide), else the LDG inter-warp kernel (P:340:
// masters = adjacent columns).  MAP_INTER_WARP_TMA falls back to the LDG
// inter-warp kernel (same result contract) where TMA cannot run.
int cudanp_tmv(const float* A, int64_t lda, const float* x, float* y, int64_t n_outer,
               int64_t n_inner, int S, int dist, int map, void* stream) {
  const bool tma = tma_ok(A, lda, n_outer, n_inner);
  if (S == CUDANP_S_AUTO) {
    if (map < CUDANP_MAP_AUTO || map > CUDANP_MAP_INTER_WARP_TMA) return fail_invalid("map");
    choose_version(0, n_outer, n_inner, tmv_aligned(A, lda, y, n_outer), tma, map, &S, &dist, &map);
  }
  const int m = map == CUDANP_MAP_INTER_WARP_TMA ? CUDANP_MAP_INTER_WARP : map;
  int rc = check_tmv_args(A, lda, x, y, n_outer, n_inner, S, dist, m);
  if (rc) return rc;
  const bool use_tma = valid_S(S) && tma &&
                       (map == CUDANP_MAP_INTER_WARP_TMA || (map == CUDANP_MAP_AUTO && tmv_wide(n_outer)));
  if (use_tma)
    return tmv_tma(A, lda, x, y, n_outer, n_inner, S, dist, 0, -1, 0, as_stream(stream), nullptr);
  return tmv_np(A, lda, x, y, n_outer, n_inner, S, dist, resolve_map(m, true, S),
                tmv_vec(A, lda, y, n_outer, n_inner, S), as_stream(stream), nullptr);
}

int cudanp_tmv_tma_ex(const float* A, int64_t lda, const float* x, float* y, int64_t n_outer,
                      int64_t n_inner, int S, int dist, int cols, int rows_sel, int stages,
                      void* stream) {
  int rc = check_tmv_args(A, lda, x, y, n_outer, n_inner, S, dist, CUDANP_MAP_INTER_WARP);
  if (rc) return rc;
  if (n_outer == 0) return CUDANP_OK;
  if (n_inner == 0)  // nothing to stream: the plain kernel writes the zeros
    return tmv_np(A, lda, x, y, n_outer, n_inner, S, dist, MAP_INTER, false, as_stream(stream), nullptr);
  if (!tma_ok(A, lda, n_outer, n_inner)) {
    set_error("TMA path needs a 16-byte aligned A, lda %% 4 == 0 and sizes < 2^31");
    return CUDANP_ERR_UNSUPPORTED;
  }
  return tmv_tma(A, lda, x, y, n_outer, n_inner, S, dist, cols, rows_sel, stages, as_stream(stream),
                 nullptr);
}

int cudanp_tmv_tma(const float* A, int64_t lda, const float* x, float* y, int64_t n_outer,
                   int64_t n_inner, int S, int dist, void* stream) {
  return cudanp_tmv_tma_ex(A, lda, x, y, n_outer, n_inner, S, dist, 0, -1, 0, stream);
}

int cudanp_mv(const float* A, int64_t lda, const float* x, float* y, int64_t n_outer,
              int64_t n_inner, int S, int dist, int map, void* stream) {
  if (S == CUDANP_S_AUTO) {
    if (map < CUDANP_MAP_AUTO || map > CUDANP_MAP_INTER_WARP) return fail_invalid("map");
    choose_version(1, n_outer, n_inner, mv_vec(A, lda, x, n_inner), false, map, &S, &dist, &map);
  }
  int rc = check_mv_args(A, lda, x, y, n_outer, n_inner, S, dist, map);
  if (rc) return rc;
  return mv_np(A, lda, x, y, n_outer, n_inner, S, dist, resolve_map(map, false, S),
               mv_vec(A, lda, x, n_inner), as_stream(stream), nullptr);
}

// out_per_item: reduce writes one value per item even when L = 0; scan
// writes N*L values, so out may be NULL when L = 0.
static int check_batched(const void* in, void* out, int64_t N, int64_t L, int S, int dist, int map,
                         int dtype, int op, bool out_per_item, bool cluster_ok = false) {
  int rc = check_common(S, dist, map, N, L, cluster_ok, cluster_ok);
  if (rc) return rc;
  rc = check_dtype_op(dtype, op);
  if (rc) return rc;
  if (N > 0 && (out_per_item || L > 0) && !out) return fail_invalid("out is NULL");
  if (N > 0 && L > 0 && !in) return fail_invalid("in is NULL");
  return CUDANP_OK;
}

int cudanp_batched_loop_reduce_tma(const void* in, const void* init, void* out, int64_t n_outer,
                                   int64_t n_inner, int dtype, int op, int S, int dist,
                                   int stage_bytes, int stages, void* stream) {
  int rc = check_batched(in, out, n_outer, n_inner, S, dist, CUDANP_MAP_INTRA_WARP, dtype, op, true);
  if (rc) return rc;
  if (!valid_S(S)) return fail_invalid("TMA-staged reduce: S must be one of 1,2,4,8,16,32");
  if (stage_bytes < 0 || stages < 0 || stages > 64) return fail_invalid("stage_bytes / stages");
  if (n_outer == 0) return CUDANP_OK;
  if (n_inner == 0)  // nothing to stream: the plain kernel writes init / the identity
    return reduce_np(in, init, out, n_outer, n_inner, dtype, op, S, dist, MAP_INTRA, false,
                     as_stream(stream), nullptr);
  if (!((n_inner % 4 == 0) && aligned16(in))) {
    set_error("TMA-staged reduce needs 16-byte aligned input and n_inner %% 4 == 0");
    return CUDANP_ERR_UNSUPPORTED;
  }
  return reduce_tma(in, init, out, n_outer, n_inner, dtype, op, S, dist, stage_bytes, stages,
                    as_stream(stream), nullptr);
}

int cudanp_batched_loop_reduce(const void* in, const void* init, void* out, int64_t n_outer,
                               int64_t n_inner, int dtype, int op, int S, int dist, int map,
                               void* stream) {
  if (map == CUDANP_MAP_INTRA_WARP_TMA && S != CUDANP_S_AUTO)
    return cudanp_batched_loop_reduce_tma(in, init, out, n_outer, n_inner, dtype, op, S, dist, 0, 0,
                                          stream);
  const bool vec = (n_inner % 4 == 0) && aligned16(in);
  if (S == CUDANP_S_AUTO) {
    if (map < CUDANP_MAP_AUTO || map > CUDANP_MAP_INTRA_WARP_TMA) return fail_invalid("map");
    if (map == CUDANP_MAP_INTRA_WARP_TMA) map = CUDANP_MAP_INTRA_WARP;
    choose_version(2, n_outer, n_inner, vec, false, map, &S, &dist, &map);
  }
  int rc = check_batched(in, out, n_outer, n_inner, S, dist, map, dtype, op, true, true);
  if (rc) return rc;
  return reduce_np(in, init, out, n_outer, n_inner, dtype, op, S, dist, resolve_map(map, false, S),
                   vec, as_stream(stream), nullptr);
}

int cudanp_batched_loop_reduce_backend(const void* in, const void* init, void* out,
                                       int64_t n_outer, int64_t n_inner, int dtype, int op, int S,
                                       int backend, void* stream) {
  int rc = check_batched(in, out, n_outer, n_inner, S, 0, CUDANP_MAP_INTRA_WARP, dtype, op, true);
  if (rc) return rc;
  if (backend < 0 || backend > 2) return fail_invalid("backend");
  if (!((n_inner % 4 == 0) && aligned16(in))) {
    set_error("backend ablation is built for the 128-bit path only (L %% 4 == 0, 16-byte aligned)");
    return CUDANP_ERR_UNSUPPORTED;
  }
  return reduce_backend(in, init, out, n_outer, n_inner, dtype, op, S, backend, as_stream(stream));
}

int cudanp_batched_loop_scan(const void* in, const void* init, void* out, int64_t n_outer,
                             int64_t n_inner, int dtype, int S, int dist, int map, void* stream) {
  const bool vec = (n_inner % 4 == 0) && aligned16(in) && aligned16(out);
  if (S == CUDANP_S_AUTO) {
    if (map < CUDANP_MAP_AUTO || map > CUDANP_MAP_INTER_WARP) return fail_invalid("map");
    choose_version(3, n_outer, n_inner, vec, false, map, &S, &dist, &map);
  }
  int rc = check_batched(in, out, n_outer, n_inner, S, dist, map, dtype, CUDANP_SUM, false, true);
  if (rc) return rc;
  return scan_np(in, init, out, n_outer, n_inner, dtype, S, dist, resolve_map(map, false, S), vec,
                 as_stream(stream), nullptr);
}

// ---------------------------------------------------------------- ragged (f1)
static int check_ragged(const void* in, const int64_t* off, void* out, int64_t N, int S, int dist,
                        int map, int dtype, int op) {
  int rc = check_common(S, dist, map, N, 0);
  if (rc) return rc;
  rc = check_dtype_op(dtype, op);
  if (rc) return rc;
  if (N > 0 && (!in || !off || !out)) return fail_invalid("in, offsets or out is NULL");
  if (((uintptr_t)off & 7u) != 0) return fail_invalid("offsets must be 8-byte aligned");
  if (((uintptr_t)in & 3u) != 0) return fail_invalid("in must be 4-byte aligned");
  return CUDANP_OK;
}

int cudanp_ragged_loop_reduce(const void* in, const int64_t* offsets, const void* init, void* out,
                              int64_t n_outer, int dtype, int op, int S, int dist, int map,
                              void* stream) {
  int rc = check_ragged(in, offsets, out, n_outer, S, dist, map, dtype, op);
  if (rc) return rc;
  return ragged_np(in, offsets, init, out, n_outer, dtype, op, S, dist, resolve_map(map, false),
                   as_stream(stream));
}

int cudanp_ragged_loop_reduce_adaptive(const void* in, const int64_t* offsets, const void* init,
                                       void* out, int64_t n_outer, int dtype, int op,
                                       int64_t threshold, void* stream) {
  int rc = check_ragged(in, offsets, out, n_outer, 1, 0, 0, dtype, op);
  if (rc) return rc;
  if (threshold < 1) return fail_invalid("threshold must be >= 1");
  return ragged_adaptive(in, offsets, init, out, n_outer, dtype, op, threshold, as_stream(stream));
}

int cudanp_ragged_loop_reduce_literal(const void* in, const int64_t* offsets, const void* init,
                                      void* out, int64_t n_outer, int dtype, int op, void* stream) {
  int rc = check_ragged(in, offsets, out, n_outer, 1, 0, 0, dtype, op);
  if (rc) return rc;
  return ragged_literal(in, offsets, init, out, n_outer, dtype, op, as_stream(stream));
}

// ---------------------------------------------------------------- LE multi-section (f2)
static int check_le(const float* in, float* gicov, int64_t N, int64_t L, int layout, int S,
                    int dist, int map) {
  if (S < 1 || S > 32) return fail_invalid("S must be one of 1,2,3,4,5,8,10,15,16,32");
  int rc = check_common(1, dist, map, N, L);
  if (rc) return rc;
  if (layout != 0 && layout != 1) return fail_invalid("layout");
  if (N > 0 && L < 1) return fail_invalid("n_inner must be >= 1 (ave = sum / L)");
  if (N > 0 && (!in || !gicov)) return fail_invalid("in or gicov is NULL");
  return CUDANP_OK;
}

int cudanp_le_gicov(const float* in, float* gicov, float* ave, float* var, float* ep,
                    int64_t n_outer, int64_t n_inner, float threshold, int layout, int S, int dist,
                    int map, void* stream) {
  int rc = check_le(in, gicov, n_outer, n_inner, layout, S, dist, map);
  if (rc) return rc;
  // MAP_AUTO: keep the masters' accesses coalesced: point-major
  // data -> inter-warp (the paper's LE choice); item-major -> intra.
  const int m = map != CUDANP_MAP_AUTO ? map : (layout ? MAP_INTER : MAP_INTRA);
  return le_np(in, gicov, ave, var, ep, n_outer, n_inner, threshold, layout, S, dist, m, false,
               as_stream(stream));
}

int cudanp_le_gicov_placement(const float* in, float* gicov, float* ave, float* var, float* ep,
                              int64_t n_outer, int64_t n_inner, float threshold, int layout, int S,
                              int dist, int map, int placement, void* stream) {
  if (placement == CUDANP_GRAD_REGISTERS)
    return cudanp_le_gicov(in, gicov, ave, var, ep, n_outer, n_inner, threshold, layout, S, dist,
                           map, stream);
  int rc = check_le(in, gicov, n_outer, n_inner, layout, S, dist, map);
  if (rc) return rc;
  const int m = map != CUDANP_MAP_AUTO ? map : (layout ? MAP_INTER : MAP_INTRA);
  if (placement == CUDANP_GRAD_GLOBAL)
    return le_np(in, gicov, ave, var, ep, n_outer, n_inner, threshold, layout, S, dist, m, true,
                 as_stream(stream));
  if (placement != CUDANP_GRAD_SHARED) return fail_invalid("placement");
  if (layout == 1) {  // point-major: inter-warp teams, one TMA box of [32 items x L points] per group
    if (m != MAP_INTER || S > 16 || n_inner > 256 || n_outer % 4 != 0 || !aligned16(in)) {
      set_error("shared-memory Grad (point-major) is built for the inter-warp map, S <= 16, "
                "n_inner <= 256, n_outer %% 4 == 0 and a 16-byte aligned input");
      return CUDANP_ERR_UNSUPPORTED;
    }
    return le_tma_pm(in, gicov, ave, var, ep, n_outer, n_inner, threshold, S, dist, as_stream(stream));
  }
  if (layout != 0 || m != MAP_INTRA || !valid_S(S) || !aligned16(in)) {
    set_error("shared-memory Grad is built for item-major data, the intra-warp map, S = 2^k <= 32 "
              "and a 16-byte aligned input");
    return CUDANP_ERR_UNSUPPORTED;
  }
  return le_tma(in, gicov, ave, var, ep, n_outer, n_inner, threshold, S, dist, as_stream(stream));
}

int cudanp_le_gicov_literal(const float* in, float* gicov, float* ave, float* var, float* ep,
                            int64_t n_outer, int64_t n_inner, float threshold, int layout,
                            void* stream) {
  int rc = check_le(in, gicov, n_outer, n_inner, layout, 1, 0, 0);
  if (rc) return rc;
  return le_literal(in, gicov, ave, var, ep, n_outer, n_inner, threshold, layout, as_stream(stream));
}

// ---------------------------------------------------------------- variants
static int check_impl(int impl) {
  if (impl != CUDANP_IMPL_S1_LITERAL && impl != CUDANP_IMPL_DP_THREAD && impl != CUDANP_IMPL_DP_BLOCK &&
      impl != CUDANP_IMPL_S1_TILED)
    return fail_invalid("impl");
  return CUDANP_OK;
}
static int tiled_unsupported() {
  set_error("the TMA-tiled S=1 baseline needs 16-byte aligned operands, rows a multiple of 4 "
            "elements and sizes < 2^31");
  return CUDANP_ERR_UNSUPPORTED;
}
static bool tiled_ok(const void* a, int64_t ld, const void* b, int64_t rows, int64_t cols) {
  return aligned16(a) && (!b || aligned16(b)) && ld % 4 == 0 && rows < (int64_t(1) << 31) &&
         cols < (int64_t(1) << 31);
}

int cudanp_tmv_variant(int impl, const float* A, int64_t lda, const float* x, float* y,
                       int64_t n_outer, int64_t n_inner, void* stream) {
  int rc = check_impl(impl);
  if (!rc) rc = check_tmv_args(A, lda, x, y, n_outer, n_inner, 1, 0, 0);
  if (rc) return rc;
  if (impl == CUDANP_IMPL_S1_LITERAL) return tmv_literal(A, lda, x, y, n_outer, n_inner, as_stream(stream));
  if (impl == CUDANP_IMPL_S1_TILED) {
    if (n_outer == 0) return CUDANP_OK;
    if (n_inner == 0) return tmv_np(A, lda, x, y, n_outer, 0, 1, 0, MAP_INTER, false, as_stream(stream), nullptr);
    if (!tma_ok(A, lda, n_outer, n_inner)) return tiled_unsupported();
    return tmv_tma(A, lda, x, y, n_outer, n_inner, 1, 0, 0, -1, 0, as_stream(stream), nullptr);
  }
  return dp_tmv(impl == CUDANP_IMPL_DP_BLOCK, A, lda, x, y, n_outer, n_inner, as_stream(stream));
}

int cudanp_mv_variant(int impl, const float* A, int64_t lda, const float* x, float* y,
                      int64_t n_outer, int64_t n_inner, void* stream) {
  int rc = check_impl(impl);
  if (!rc) rc = check_mv_args(A, lda, x, y, n_outer, n_inner, 1, 0, 0);
  if (rc) return rc;
  if (impl == CUDANP_IMPL_S1_LITERAL) return mv_literal(A, lda, x, y, n_outer, n_inner, as_stream(stream));
  if (impl == CUDANP_IMPL_S1_TILED) {
    if (n_outer > 0 && n_inner > 0 && !(tiled_ok(A, lda, x, n_outer, n_inner) && n_inner % 4 == 0))
      return tiled_unsupported();  // (x chunks are 1-D bulk copies: 16-byte aligned, w % 4 == 0)
    return mv_s1_tiled(A, lda, x, y, n_outer, n_inner, as_stream(stream));
  }
  return dp_mv(impl == CUDANP_IMPL_DP_BLOCK, A, lda, x, y, n_outer, n_inner, as_stream(stream));
}

int cudanp_batched_loop_reduce_variant(int impl, const void* in, const void* init, void* out,
                                       int64_t n_outer, int64_t n_inner, int dtype, int op,
                                       void* stream) {
  int rc = check_impl(impl);
  if (!rc) rc = check_batched(in, out, n_outer, n_inner, 1, 0, 0, dtype, op, true);
  if (rc) return rc;
  if (impl == CUDANP_IMPL_S1_LITERAL)
    return reduce_literal(in, init, out, n_outer, n_inner, dtype, op, as_stream(stream));
  if (impl == CUDANP_IMPL_S1_TILED) {
    if (n_outer > 0 && n_inner == 0)  // nothing to stream: init / the identity
      return reduce_np(in, init, out, n_outer, 0, dtype, op, 1, 0, MAP_INTRA, false, as_stream(stream), nullptr);
    if (n_outer > 0 && !tiled_ok(in, n_inner, nullptr, n_outer, n_inner)) return tiled_unsupported();
    return reduce_s1_tiled(in, init, out, n_outer, n_inner, dtype, op, as_stream(stream));
  }
  return dp_reduce(impl == CUDANP_IMPL_DP_BLOCK, in, init, out, n_outer, n_inner, dtype, op,
                   as_stream(stream));
}

int cudanp_batched_loop_scan_variant(int impl, const void* in, const void* init, void* out,
                                     int64_t n_outer, int64_t n_inner, int dtype, void* stream) {
  int rc = check_impl(impl);
  if (!rc) rc = check_batched(in, out, n_outer, n_inner, 1, 0, 0, dtype, CUDANP_SUM, false);
  if (rc) return rc;
  if (impl == CUDANP_IMPL_S1_LITERAL)
    return scan_literal(in, init, out, n_outer, n_inner, dtype, as_stream(stream));
  if (impl == CUDANP_IMPL_S1_TILED) {
    if (n_outer > 0 && n_inner > 0 && !tiled_ok(in, n_inner, out, n_outer, n_inner)) return tiled_unsupported();
    return scan_s1_tiled(in, init, out, n_outer, n_inner, dtype, as_stream(stream));
  }
  return dp_scan(impl == CUDANP_IMPL_DP_BLOCK, in, init, out, n_outer, n_inner, dtype,
                 as_stream(stream));
}

int cudanp_dp_set_pending_launch_limit(size_t n) {
  if (cudaDeviceSetLimit(cudaLimitDevRuntimePendingLaunchCount, n) != cudaSuccess)
    return check_launch("cudaDeviceSetLimit(DevRuntimePendingLaunchCount)");
  return CUDANP_OK;
}

int cudanp_dp_error_count(int reset, int64_t* count_out) { return dp_error_count(reset, count_out); }

int cudanp_dp_memcopy(const float* in, float* out, int64_t total, int64_t m, int variant,
                      void* stream) {
  if (total < 0 || (total > 0 && (!in || !out))) return fail_invalid("memcopy sizes/pointers");
  if (variant < 0 || variant > 2) return fail_invalid("memcopy variant");
  if (variant == 2 && (m < 1 || total % m != 0)) return fail_invalid("m must divide total");
  if (total == 0) return CUDANP_OK;
  if (variant == 0) {
    memcopy_kernel<<<(unsigned)(sm_count() * 8), 256, 0, as_stream(stream)>>>(in, out, total);
    return check_launch("memcopy launch");
  }
  return dp_memcopy(in, out, total, m, variant, as_stream(stream));
}

// ---------------------------------------------------------------- launch info
int cudanp_launch_info(int op_kind, int64_t n_outer, int64_t n_inner, int dtype, int op, int S,
                       int dist, int map, int vec4, int* block_threads, int64_t* grid_ctas,
                       int* regs_per_thread, int* smem_bytes, int* resolved_map, int* S_used,
                       int* dist_used) {
  const bool v = vec4 != 0;
  if (S == CUDANP_S_AUTO && op_kind >= 0 && op_kind <= 3) {
    if (map < CUDANP_MAP_AUTO || map > (op_kind == 0 ? CUDANP_MAP_INTER_WARP_TMA : CUDANP_MAP_INTER_WARP))
      return fail_invalid("map");
    choose_version(op_kind, n_outer, n_inner, v, v, map, &S, &dist, &map);
  }
  // TMV: MAP_AUTO / MAP_INTER_WARP_TMA resolve as cudanp_tmv does (vec4 stands
  // for the TMA preconditions).
  if (op_kind == 0 && valid_S(S) && v && n_outer > 0 && n_inner > 0 &&
      (map == CUDANP_MAP_INTER_WARP_TMA || (map == CUDANP_MAP_AUTO && tmv_wide(n_outer))))
    op_kind = 4;
  if (op_kind == 0 && map == CUDANP_MAP_INTER_WARP_TMA) map = CUDANP_MAP_INTER_WARP;
  if (op_kind == 4) map = CUDANP_MAP_INTER_WARP;
  int rc = check_common(S, dist, map, n_outer, n_inner, op_kind >= 1 && op_kind <= 3,
                        op_kind <= 3);
  if (rc) return rc;
  LaunchInfo info;
  const int m = resolve_map(map, op_kind == 0, S);
  switch (op_kind) {
    case 0:  // vec4 = aligned; the call adds its shape rule (tmv_vec)
      rc = tmv_np(nullptr, 0, nullptr, nullptr, n_outer, n_inner, S, dist, m,
                  v && tmv_vec_shape(n_outer, n_inner, S), 0, &info);
      break;
    case 1: rc = mv_np(nullptr, 0, nullptr, nullptr, n_outer, n_inner, S, dist, m, v, 0, &info); break;
    case 2:
      rc = check_dtype_op(dtype, op);
      if (!rc) rc = reduce_np(nullptr, nullptr, nullptr, n_outer, n_inner, dtype, op, S, dist, m, v, 0, &info);
      break;
    case 3:
      rc = check_dtype_op(dtype, CUDANP_SUM);
      if (!rc) rc = scan_np(nullptr, nullptr, nullptr, n_outer, n_inner, dtype, S, dist, m, v, 0, &info);
      break;
    case 4:  // TMA-staged TMV (auto shape), inter-warp
      if (n_outer == 0 || n_inner == 0) return fail_invalid("tma launch shape needs n_outer, n_inner > 0");
      rc = tmv_tma(nullptr, 0, nullptr, nullptr, n_outer, n_inner, S, dist, 0, -1, 0, 0, &info);
      break;
    case 5:  // TMA-staged reduce (auto shape), intra-warp
      if (n_outer == 0 || n_inner == 0 || n_inner % 4) return fail_invalid("tma reduce shape needs N, L > 0, L % 4 == 0");
      rc = check_dtype_op(dtype, op);
      if (!rc) rc = reduce_tma(nullptr, nullptr, nullptr, n_outer, n_inner, dtype, op, S, dist, 0, 0, 0, &info);
      break;
    default: return fail_invalid("op_kind");
  }
  if (rc) return rc;
  if (block_threads) *block_threads = info.block_threads;
  if (grid_ctas) *grid_ctas = info.grid;
  if (regs_per_thread) *regs_per_thread = info.regs;
  if (smem_bytes) *smem_bytes = info.smem;
  if (resolved_map) *resolved_map = op_kind == 4 ? CUDANP_MAP_INTER_WARP_TMA : info.map;
  if (S_used) *S_used = S;
  if (dist_used) *dist_used = dist;
  return CUDANP_OK;
}

int cudanp_choose_version(int op_kind, int64_t n_outer, int64_t n_inner, int vec4, int map, int* S,
                          int* dist, int* map_out) {
  if (op_kind < 0 || op_kind > 3) return fail_invalid("op_kind");
  if (n_outer < 0 || n_inner < 0) return fail_invalid("negative size");
  if (map < CUDANP_MAP_AUTO || map > (op_kind == 0 ? CUDANP_MAP_INTER_WARP_TMA : CUDANP_MAP_INTER_WARP))
    return fail_invalid("map");
  if (!S || !dist || !map_out) return fail_invalid("NULL output");
  return choose_version(op_kind, n_outer, n_inner, vec4 != 0, vec4 != 0, map, S, dist, map_out);
}

// ---------------------------------------------------------------- CUDA IPC (f4)
// cuMemGetAddressRange through the runtime's driver entry point, so the
// library needs no link-time libcuda (it must load on GPU-less build hosts).
typedef int (*MemGetAddressRangeFn)(unsigned long long*, size_t*, unsigned long long);

static int alloc_base(const void* ptr, char** base) {
  static MemGetAddressRangeFn fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) != cudaSuccess ||
        !f) {
      cudaGetLastError();
      set_error("cuMemGetAddressRange entry point unavailable");
      return CUDANP_ERR_CUDA;
    }
    fn = (MemGetAddressRangeFn)f;
  }
  unsigned long long b = 0;
  size_t sz = 0;
  if (fn(&b, &sz, (unsigned long long)(uintptr_t)ptr) != 0) {
    set_error("cuMemGetAddressRange failed (not a device allocation?)");
    return CUDANP_ERR_CUDA;
  }
  *base = (char*)(uintptr_t)b;
  return CUDANP_OK;
}

int cudanp_ipc_get_handle(const void* dev_ptr, void* handle_out, int64_t* offset_out) {
  if (!dev_ptr || !handle_out || !offset_out) return fail_invalid("ipc_get_handle arguments");
  char* base = nullptr;
  int rc = alloc_base(dev_ptr, &base);
  if (rc) return rc;
  cudaIpcMemHandle_t h;
  if (cudaIpcGetMemHandle(&h, base) != cudaSuccess) return check_launch("cudaIpcGetMemHandle");
  memcpy(handle_out, &h, sizeof(h));
  *offset_out = (int64_t)((const char*)dev_ptr - base);
  return CUDANP_OK;
}

int cudanp_ipc_open(const void* handle, int64_t offset, void** dev_ptr_out) {
  if (!handle || !dev_ptr_out || offset < 0) return fail_invalid("ipc_open arguments");
  cudaIpcMemHandle_t h;
  memcpy(&h, handle, sizeof(h));
  void* base = nullptr;
  if (cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess)
    return check_launch("cudaIpcOpenMemHandle");
  *dev_ptr_out = (char*)base + offset;
  return CUDANP_OK;
}

int cudanp_ipc_close(void* dev_ptr, int64_t offset) {
  if (!dev_ptr || offset < 0) return fail_invalid("ipc_close arguments");
  if (cudaIpcCloseMemHandle((char*)dev_ptr - offset) != cudaSuccess)
    return check_launch("cudaIpcCloseMemHandle");
  return CUDANP_OK;
}

// ---------------------------------------------------------------- sharding
int cudanp_shard_range(int64_t n_outer, int nranks, int rank, int64_t* begin, int64_t* end) {
  if (n_outer < 0 || nranks < 1 || rank < 0 || rank >= nranks || !begin || !end)
    return fail_invalid("shard_range arguments");
  *begin = (int64_t)(((__int128)rank * n_outer) / nranks);
  *end = (int64_t)(((__int128)(rank + 1) * n_outer) / nranks);
  return CUDANP_OK;
}

// ---------------------------------------------------------------- test support
int cudanp_generate(void* out, int64_t rows, int64_t cols, int64_t ld, int64_t row0, int64_t col0,
                    int64_t w_global, int stream_id, int kind, int64_t B, uint64_t seed,
                    void* stream) {
  if (rows < 0 || cols < 0 || ld < cols || row0 < 0 || col0 < 0 || w_global < 0)
    return fail_invalid("generate sizes");
  if (kind < 0 || kind > 6) return fail_invalid("generate kind");
  if (kind == 3 && (B < 1 || (B & (B - 1)))) return fail_invalid("generate B must be a power of two");
  if (rows * cols == 0) return CUDANP_OK;
  if (!out) return fail_invalid("generate out is NULL");
  const uint64_t key = mix64(seed ^ ((uint64_t)stream_id << 56));
  const int64_t total = rows * cols;
  int64_t grid = (total + 255) / 256;
  const int64_t cap = (int64_t)sm_count() * 16;
  if (grid > cap) grid = cap;
  generate_kernel<<<(unsigned)grid, 256, 0, as_stream(stream)>>>(out, rows, cols, ld, row0, col0,
                                                                 w_global, key, kind, B);
  return check_launch("generate launch");
}

}  // extern "C"

extern "C" {

static int copy_back(void* dst, const void* src, size_t bytes, const char* what) {
  if (cudaDeviceSynchronize() != cudaSuccess) return check_launch(what);
  if (cudaMemcpy(dst, src, bytes, cudaMemcpyDeviceToHost) != cudaSuccess) return check_launch(what);
  return CUDANP_OK;
}

int cudanp_debug_owner_map(int64_t n_inner, int S, int dist, int V, int32_t* owner_host) {
  if (!valid_S(S) || (dist != 0 && dist != 1) || (V != 1 && V != 4) || n_inner < 0 ||
      n_inner > (1 << 26) || (n_inner > 0 && !owner_host))
    return fail_invalid("debug_owner_map arguments");
  if (n_inner == 0) return CUDANP_OK;
  int32_t* d = nullptr;
  if (cudaMalloc(&d, n_inner * sizeof(int32_t)) != cudaSuccess) return check_launch("cudaMalloc");
  cudaMemset(d, 0xff, n_inner * sizeof(int32_t));
  CUDANP_DISPATCH_S(S, {
    if (dist == DIST_CYCLIC) owner_kernel<kS, DIST_CYCLIC><<<1, kS>>>(n_inner, V, d);
    else owner_kernel<kS, DIST_BLOCK><<<1, kS>>>(n_inner, V, d);
  });
  int rc = copy_back(owner_host, d, n_inner * sizeof(int32_t), "debug_owner_map");
  cudaFree(d);
  return rc;
}

int cudanp_debug_team_ids(int S, int map, int32_t* master_host, int32_t* slave_host, int* nthreads) {
  if (!valid_S(S) || (map != CUDANP_MAP_INTRA_WARP && map != CUDANP_MAP_INTER_WARP) ||
      !master_host || !slave_host || !nthreads)
    return fail_invalid("debug_team_ids arguments");
  const int n = map == CUDANP_MAP_INTRA_WARP ? 64 : 32 * S;
  int32_t* d = nullptr;
  if (cudaMalloc(&d, 2 * n * sizeof(int32_t)) != cudaSuccess) return check_launch("cudaMalloc");
  CUDANP_DISPATCH_S(S, {
    if (map == CUDANP_MAP_INTRA_WARP) team_intra_kernel<kS><<<1, 64>>>(d, d + n);
    else team_inter_kernel<kS><<<1, dim3(32, kS)>>>(d, d + n);
  });
  int rc = copy_back(master_host, d, n * sizeof(int32_t), "debug_team_ids");
  if (!rc) rc = copy_back(slave_host, d + n, n * sizeof(int32_t), "debug_team_ids");
  cudaFree(d);
  *nthreads = n;
  return rc;
}

int cudanp_debug_broadcast(int S, int map, int32_t* out_host, int* nthreads) {
  if (!valid_S(S) || (map != CUDANP_MAP_INTRA_WARP && map != CUDANP_MAP_INTER_WARP) || !out_host ||
      !nthreads)
    return fail_invalid("debug_broadcast arguments");
  const int n = map == CUDANP_MAP_INTRA_WARP ? 64 : 32 * S;
  int32_t* d = nullptr;
  if (cudaMalloc(&d, n * sizeof(int32_t)) != cudaSuccess) return check_launch("cudaMalloc");
  CUDANP_DISPATCH_S(S, {
    if (map == CUDANP_MAP_INTRA_WARP) bcast_intra_kernel<kS><<<1, 64>>>(d);
    else bcast_inter_kernel<kS><<<1, dim3(32, kS)>>>(d);
  });
  int rc = copy_back(out_host, d, n * sizeof(int32_t), "debug_broadcast");
  cudaFree(d);
  *nthreads = n;
  return rc;
}

}  // extern "C"
