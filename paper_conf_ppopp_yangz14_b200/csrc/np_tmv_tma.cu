// np_tmv_tma.cu -- TMV with TMA-staged tiles (the north star's "TMA or
// cp.async staging where the access pattern is strided (as in y=A^T x)").
//
// Same method as tmv_inter_kernel (Fig 2; inter-warp NP):
// a CTA owns COLS = 32 x V column-masters' outputs (V per lane) and S slave
// warps share the rows, cyclic or block (R5); the S partials meet in
// shared memory and the master warp stores.  What changes is
// how A reaches the slaves: instead of each lane issuing 128-bit loads, one
// elected thread streams [rows x COLS columns] tiles of A into a ring of
// shared-memory stages with the Tensor Memory Accelerator
// (cp.async.bulk.tensor.2d, completion counted on an mbarrier), and the
// slaves read their rows from shared memory.  Memory-level parallelism then
// comes from the stages in flight, not from the number of resident threads.
//
//  cyclic: one box of R rows per stage (TmaShape); slave s owns the box rows
//          k*S + s, i.e. global rows i = s (mod S) exactly as P:166.
//  block : S boxes of R/S rows per stage, one from each slave's contiguous
//          chunk [s*c, (s+1)*c) (c = ceil(h/S)).  When S divides h the
//          tensor map views A as [S chunks][c rows][w columns] and the S
//          boxes are one 3-D box, one copy instruction per stage (box3d).
// Rows past h come back zero-filled by TMA and are masked before x is read.
// A block stage's box may run past the slave's chunk into the next slave's
// rows (RK need not divide c); those rows are skipped (no FMA), so a
// non-finite value there cannot leak into this slave's sum.
#include <cuda.h>

#include "common.cuh"
#include "np_team.cuh"
#include "np_tma.cuh"

namespace cudanp {

// Launch shape.  Rows per slave per stage RK comes in three sizes per S (a
// stage holds R = RK x S rows; a cyclic box is R rows <= 256 = the TMA box
// limit, a block stage is S boxes of RK rows); the ring depth is a runtime
// value (see tma_shape below).
template <int S> struct TmaRK {
  static constexpr int v0 = S == 1 ? 32 : (S <= 4 ? 16 : 128 / S / 2);
  static constexpr int v1 = 2 * v0;
  static constexpr int v2 = 4 * v0;
  static constexpr int get(int sel) { return sel == 0 ? v0 : (sel == 1 ? v1 : v2); }
};
// A dedicated producer warp needs 32 more threads than the team: S <= 16.
template <int S> struct TmaPW { static constexpr bool value = S < 32; };
template <int S> struct TmaThreads { static constexpr int value = 32 * S + (TmaPW<S>::value ? 32 : 0); };
// CTAs per SM the register budget guarantees (and the most the shape policy
// counts on): 4 for S <= 8, 2 for S = 16 (60 registers), 1 for S = 32 (a
// 1024-thread CTA keeps 64 registers rather than spill at 32).
template <int S> struct TmaMinBlocks {
  static constexpr int value = S >= 32 ? 1 : (S == 16 ? 2 : 4);
};

// COLS = columns per CTA = 32 lanes x V (V = 4, 2, 1).  Warps 0..S-1 are the
// team (slave warp s; warp 0's lanes are the masters); with PW, warp S is a
// dedicated producer whose lane 0 only issues TMA copies, so a slow slave
// never delays the refill of a stage the others are done with.  Without PW
// (S = 32: a 33rd warp would exceed 1024 threads) thread 0 refills, one tile
// behind its own consumption, the stage every slave has already released.
template <int S, int DIST, int COLS, int RK>
__global__ void __launch_bounds__(TmaThreads<S>::value, TmaMinBlocks<S>::value)
tmv_tma_kernel(const __grid_constant__ CUtensorMap mapA, const float* __restrict__ x,
               float* __restrict__ y, int64_t w, int64_t h, int stages, int box3d) {
  pdl_entry();
  constexpr bool PW = TmaPW<S>::value;
  constexpr int V = COLS / 32;
  constexpr int R = RK * S;  // rows per stage
  static_assert(R <= 256 || DIST == DIST_BLOCK, "TMA box height <= 256");
  static_assert(RK <= 256, "TMA box height <= 256");
  extern __shared__ __align__(128) unsigned char smem_raw[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw);             // [stages]
  uint64_t* empty = full + stages;                                    // [stages]
  float* tiles = reinterpret_cast<float*>(smem_raw + 128 * ((16 * stages + 127) / 128));  // [stages][R][COLS]
  float* red = tiles;                                                 // [S][COLS], reused after the loop

  const int lane = threadIdx.x & 31, s = threadIdx.x >> 5;            // master lane, slave warp
  const int col0 = blockIdx.x * COLS;
  const int64_t c = (h + S - 1) / S;                                  // block: rows per chunk
  const int ntiles = (int)((c + RK - 1) / RK);                        // both: rows per slave / RK
  const uint32_t stage_bytes = R * COLS * 4;

  if (threadIdx.x == 0) {
    for (int i = 0; i < stages; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], S);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  auto issue = [&](int t) {
    const int st = t % stages;
    float* dst = tiles + st * R * COLS;
    mbar_expect_tx(&full[st], stage_bytes);
    if (DIST == DIST_CYCLIC) {
      tma_load_2d(dst, &mapA, col0, t * R, &full[st]);
    } else if (box3d) {
      tma_load_3d(dst, &mapA, col0, t * RK, 0, &full[st]);
    } else {
      for (int k = 0; k < S; ++k)
        tma_load_2d(dst + k * RK * COLS, &mapA, col0, (int)(k * c + (int64_t)t * RK), &full[st]);
    }
  };

  V4<float> acc = {0.f, 0.f, 0.f, 0.f};
  if (PW && s == S) {
    // ---- producer warp: fill the ring, then refill each stage once every
    // slave has released it.
    if (lane == 0) {
      for (int t = 0; t < ntiles; ++t) {
        if (t >= stages) mbar_wait(&empty[t % stages], ((t / stages) - 1) & 1);
        issue(t);
      }
    }
  } else {
    if (!PW && threadIdx.x == 0)
      for (int t = 0; t < stages && t < ntiles; ++t) issue(t);
    for (int t = 0; t < ntiles; ++t) {
      const int st = t % stages;
      // x does not depend on the TMA: issue its loads before waiting on the
      // stage so their latency hides behind the tile's arrival.  Tall block
      // shares (RK > 16) take x 16 rows at a time, the next chunk's loads in
      // flight during this chunk's FMAs, so the x registers never outgrow
      // the budget (RK = 32-128 block spilled 200-424 bytes).
      constexpr int XC = DIST == DIST_BLOCK && RK > 16 ? 16 : RK;
      // block: is every row of this tile inside the slave's chunk and below h?
      const bool whole = DIST == DIST_CYCLIC ||
                         ((int64_t)(t + 1) * RK <= c && s * c + (int64_t)(t + 1) * RK <= h);
      const float* tile = tiles + st * R * COLS;
      auto load_x = [&](float (&xs)[XC], int k0) {
#pragma unroll
        for (int j = 0; j < XC; ++j) {
          const int kk = k0 + j;
          int64_t row;
          bool ok;
          if (DIST == DIST_CYCLIC) {
            row = (int64_t)t * R + kk * S + s;   // i = slave_id + k*slave_size
            ok = row < h;
          } else {
            const int64_t k = (int64_t)t * RK + kk;
            row = s * c + k;                    // R5: slave s owns [s*c, (s+1)*c)
            ok = k < c && row < h;
          }
          xs[j] = ok ? __ldg(x + row) : 0.f;
        }
      };
      auto fma_rows = [&](const float (&xs)[XC], int k0) {
#pragma unroll
        for (int j = 0; j < XC; ++j) {
          const int kk = k0 + j;
          const int lr = DIST == DIST_CYCLIC ? kk * S + s : s * RK + kk;
          const float xv = xs[j];
          if (DIST == DIST_BLOCK && !whole) {  // ragged last tile: skip rows outside the chunk
            const int64_t k = (int64_t)t * RK + kk;
            if (!(k < c && s * c + k < h)) continue;
          }
          const float* ap = tile + lr * COLS + lane * V;
          if constexpr (V == 4) {
            const float4 a = *reinterpret_cast<const float4*>(ap);
            acc.x = fmaf(a.x, xv, acc.x); acc.y = fmaf(a.y, xv, acc.y);
            acc.z = fmaf(a.z, xv, acc.z); acc.w = fmaf(a.w, xv, acc.w);
          } else if constexpr (V == 2) {
            const float2 a = *reinterpret_cast<const float2*>(ap);
            acc.x = fmaf(a.x, xv, acc.x); acc.y = fmaf(a.y, xv, acc.y);
          } else {
            acc.x = fmaf(*ap, xv, acc.x);
          }
        }
      };
      float xa[XC];
      load_x(xa, 0);
      mbar_wait(&full[st], (t / stages) & 1);
      if constexpr (XC == RK) {
        fma_rows(xa, 0);
      } else {
#pragma unroll
        for (int k0 = 0; k0 < RK; k0 += XC) {
          const bool more = k0 + XC < RK;
          float xb[XC];
          if (more) load_x(xb, k0 + XC);
          fma_rows(xa, k0);
          if (more) {
#pragma unroll
            for (int j = 0; j < XC; ++j) xa[j] = xb[j];
          }
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[st]);      // this slave is done with the stage
      if (!PW && threadIdx.x == 0 && t >= 1 && t - 1 + stages < ntiles) {
        const int tp = t - 1;                      // refill the stage of tile t-1
        mbar_wait(&empty[tp % stages], (tp / stages) & 1);
        issue(tp + stages);
      }
    }
  }
  // Team reduction through shared memory (the ring is free once every slave
  // is past its last tile); the master warp folds the partials in slave order.
  __syncthreads();
  if (s < S) {
    float* rr = red + s * COLS + lane * V;
    const float av[4] = {acc.x, acc.y, acc.z, acc.w};
#pragma unroll
    for (int v = 0; v < V; ++v) rr[v] = av[v];
  }
  __syncthreads();
  if (s == 0) {
    const int64_t col = col0 + lane * V;
    float sum[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
    for (int k = 0; k < S; ++k) {
      const float* p = red + k * COLS + lane * V;
#pragma unroll
      for (int v = 0; v < V; ++v) sum[v] += p[v];
    }
#pragma unroll
    for (int v = 0; v < V; ++v)
      if (col + v < w) y[col + v] = sum[v];
  }
}

// ---------------------------------------------------------------- host side
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess)
      fn = (EncodeTiledFn)f;
    else
      cudaGetLastError();
  }
  return fn;
}

static size_t tma_header_bytes(int stages) { return 128 * ((16 * (size_t)stages + 127) / 128); }

template <int S, int DIST, int COLS, int RK>
static int launch_tmv_tma_s(const float* A, int64_t lda, const float* x, float* y, int64_t w,
                            int64_t h, int stages, cudaStream_t st, LaunchInfo* info) {
  constexpr int R = RK * S;
  const size_t tile_bytes = (size_t)R * COLS * 4;
  const size_t smem = tma_header_bytes(stages) + (size_t)stages * tile_bytes;
  auto kern = tmv_tma_kernel<S, DIST, COLS, RK>;
  const unsigned grid = (unsigned)((w + COLS - 1) / COLS);
  if (info) {
    info->block_threads = TmaThreads<S>::value;
    info->grid = grid;
    info->smem = (int)smem;
    info->map = MAP_INTER;
    kernel_attrs(kern, &info->regs, nullptr);
    return CUDANP_OK;
  }
  EncodeTiledFn enc = encode_fn();
  if (!enc) {
    set_error("cuTensorMapEncodeTiled entry point unavailable");
    return CUDANP_ERR_CUDA;
  }
  CUtensorMap map;
  // block distribution with S | h: A as [S][h/S][w], one 3-D box of RK rows
  // from every chunk per stage
  const int box3d = DIST == DIST_BLOCK && S > 1 && h % S == 0 ? 1 : 0;
  const cuuint64_t c = (cuuint64_t)(h / S);
  const cuuint64_t dims[3] = {(cuuint64_t)w, box3d ? c : (cuuint64_t)h, (cuuint64_t)S};
  const cuuint64_t strides[2] = {(cuuint64_t)lda * 4, c * (cuuint64_t)lda * 4};
  const cuuint32_t box[3] = {(cuuint32_t)COLS, DIST == DIST_CYCLIC ? (cuuint32_t)R : (cuuint32_t)RK,
                             (cuuint32_t)S};
  const cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, box3d ? 3 : 2, (void*)A, dims, strides, box,
                   estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    set_error("cuTensorMapEncodeTiled failed (%d)", (int)r);
    return CUDANP_ERR_CUDA;
  }
  if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) != cudaSuccess)
    return check_launch("tmv_tma smem attribute");
  launch_pdl(kern, dim3(grid), dim3(TmaThreads<S>::value), smem, st, map, x, y, w, h, stages, box3d);
  return check_launch("tmv_tma launch");
}

// Shared memory of one SM that resident CTAs can take (B200: 228 KB per SM,
// 1 KB reserved per CTA, <= 227 KB per CTA).
static constexpr size_t kSmemPerSM = 228 * 1024, kSmemPerCTA = 227 * 1024, kSmemReserve = 1024;

// Launch shape for the TMA TMV (measured on C2, profiles/tma_explore_*.jsonl).
// The unit of work is a column strip (COLS columns, every row), so the grid
// is ceil(w / COLS) CTAs of equal work.  What matters most is the size of a
// stage: 32-64 KB boxes (R ~ 128 rows of 256-512 B) stream at 6.3-6.8 TB/s,
// 4-8 KB boxes at 3-4.6 TB/s, whatever the ring depth.  Second, the grid
// should be resident at once (3.5 waves of 1-CTA-per-SM strips lose a sixth
// of the time to the last wave), while a grid slightly smaller than the SM
// count costs little (128 SMs still pull the full HBM bandwidth).  So: among
// strip widths with >= 0.8 x SMs strips, RK options and ring depths that fit,
// prefer (all resident, >= 3 stages, R <= 128, largest stage <= 64 KB, widest
// strip).
struct TmaShapeSel {
  int cols, rk_sel, stages;
};
template <int S>
static TmaShapeSel tma_shape(int64_t w, int dist, int cols_req, int rk_req, int stages_req) {
  const int sms = sm_count();
  const int threads = TmaThreads<S>::value;
  TmaShapeSel best{0, 0, 0};
  long best_score = -1;
  const int cands[3] = {128, 64, 32};
  for (int ci = 0; ci < 3; ++ci) {
    const int cols = cands[ci];
    if (cols_req && cols != cols_req) continue;
    const int64_t grid = (w + cols - 1) / cols;
    if (!cols_req && cols > 32 && grid * 5 < (int64_t)sms * 4) continue;
    const int64_t need = (grid + sms - 1) / sms;
    const int64_t max_per_sm = S >= 16 ? TmaMinBlocks<S>::value : 2048 / threads < 8 ? 2048 / threads : 8;
    const bool resident = need <= max_per_sm;
    const int64_t per_sm = resident ? need : max_per_sm;
    size_t budget = kSmemPerSM / (size_t)per_sm;
    budget = budget > kSmemReserve + 128 ? budget - kSmemReserve - 128 : 0;
    if (budget > kSmemPerCTA - 128) budget = kSmemPerCTA - 128;
    for (int rs = 0; rs < 3; ++rs) {
      if (rk_req >= 0 && rs != rk_req) continue;
      const int R = TmaRK<S>::get(rs) * S;
      if (dist == DIST_CYCLIC && R > 256) continue;
      const size_t tile = (size_t)R * cols * 4;
      int stages = (int)(budget / tile);
      if (stages > 8) stages = 8;
      if (stages_req) stages = stages_req;
      if (stages < 2 || tma_header_bytes(stages) + stages * tile > kSmemPerCTA) continue;
      const long score = ((long)resident << 40) | ((long)(stages >= 3) << 39) | ((long)(R <= 128) << 38) |
                         ((long)(tile <= 65536 ? tile : 0) << 8) | (long)cols;
      if (score > best_score) {
        best_score = score;
        best = {cols, rs, stages};
      }
    }
  }
  return best;
}

template <int S, int DIST>
static int tmv_tma_dispatch(const float* A, int64_t lda, const float* x, float* y, int64_t w,
                            int64_t h, int cols_req, int rk_req, int stages_req, cudaStream_t st,
                            LaunchInfo* info) {
  const TmaShapeSel sel = tma_shape<S>(w, DIST, cols_req, rk_req, stages_req);
  if (!sel.cols) return fail_invalid("tmv_tma: no launch shape fits (cols / rows_sel / stages)");
#define CUDANP_TMA_RK(C)                                                                           \
  switch (sel.rk_sel) {                                                                            \
    case 0: return launch_tmv_tma_s<S, DIST, C, TmaRK<S>::v0>(A, lda, x, y, w, h, sel.stages, st, info); \
    case 1: return launch_tmv_tma_s<S, DIST, C, TmaRK<S>::v1>(A, lda, x, y, w, h, sel.stages, st, info); \
    default:                                                                                       \
      if constexpr (DIST == DIST_BLOCK || TmaRK<S>::v2 * S <= 256)                                 \
        return launch_tmv_tma_s<S, DIST, C, TmaRK<S>::v2>(A, lda, x, y, w, h, sel.stages, st, info); \
      return fail_invalid("tmv_tma: cyclic box taller than 256 rows");                             \
  }
  if (sel.cols == 128) { CUDANP_TMA_RK(128) }
  if (sel.cols == 64) { CUDANP_TMA_RK(64) }
  CUDANP_TMA_RK(32)
#undef CUDANP_TMA_RK
}

// Preconditions (checked by the ABI): A 16-byte aligned, lda % 4 == 0,
// h and w < 2^31 (TMA coordinates are int32).  cols (0 = auto, else 32, 64,
// 128), rk_sel (-1 = auto, 0/1/2 = TmaRK v0/v1/v2) and stages (0 = auto, >= 2) are
// tuning knobs; info != nullptr only fills the launch shape.
int tmv_tma(const float* A, int64_t lda, const float* x, float* y, int64_t w, int64_t h, int S,
            int dist, int cols, int rk_sel, int stages, cudaStream_t st, LaunchInfo* info) {
  if (w == 0) return CUDANP_OK;
  if (!(cols == 0 || cols == 32 || cols == 64 || cols == 128)) return fail_invalid("tma cols");
  if (rk_sel < -1 || rk_sel > 2) return fail_invalid("tma rows-per-slave selector");
  if (stages < 0 || stages > 64) return fail_invalid("tma stages");
  CUDANP_DISPATCH_S(S, {
    return dist == DIST_CYCLIC
               ? tmv_tma_dispatch<kS, DIST_CYCLIC>(A, lda, x, y, w, h, cols, rk_sel, stages, st, info)
               : tmv_tma_dispatch<kS, DIST_BLOCK>(A, lda, x, y, w, h, cols, rk_sel, stages, st, info);
  });
  return CUDANP_OK;
}

}  // namespace cudanp
