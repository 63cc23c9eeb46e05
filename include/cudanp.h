/*
 * cudanp.h -- C ABI of the B200-native CUDA-NP hot path (libcudanp.so).
 *
 * Paper: Y. Yang, H. Zhou, "CUDA-NP: Realizing Nested Thread-Level
 * Parallelism in GPGPU Applications", PPoPP'14.  "P:n" = line n of the
 * paper text; "Rn" = reading n in DESIGN.md.
 *
 * The problem: N independent outer work items
 * (the original GPU threads, "masters"), each running sequential code plus a
 * parallel inner loop of runtime trip count L with an optional
 * reduction or scan.  Each call runs hand-written sm_100a
 * master/slave kernels: a team of S threads (S counts the master, P:180;
 * S in {1,2,4,8,16,32}) shares each item's loop, with
 *   dist: CUDANP_DIST_CYCLIC or CUDANP_DIST_BLOCK (R5), and
 *   map : CUDANP_MAP_INTRA_WARP (team = S lanes of one warp) or
 *         CUDANP_MAP_INTER_WARP (team = one lane in each of S warps)
 *         (P:189-191), CUDANP_MAP_AUTO choosing per the rules of P:340-342.
 * S = 1 means no nesting: the tuned one-thread-per-item kernel.
 * S in {3, 5, 10, 15} (Fig 12; "for inter-warp NP, such
 * limitation can be removed"): teams that are not a power of two, built for
 * the inter-warp map of the four hot-path calls (and cudanp_le_gicov);
 * CUDANP_MAP_AUTO resolves to inter-warp for them, CUDANP_MAP_INTRA_WARP
 * returns CUDANP_ERR_UNSUPPORTED.
 * S = CUDANP_S_AUTO (0): the library chooses (S, dist, map) for the shape
 * (cudanp_choose_version; `dist` is then ignored, `map` kept unless AUTO) --
 * the paper's version selection as a rule distilled from the
 * B200 sweeps, with no timing at call time (cudanp_autotune times them).
 * S in {64, 128, 256, 512, 1024} ("shared-memory fallback when S exceeds
 * 32"): a team of S/32 consecutive warps, shfl inside each warp and shared
 * memory across them; supported by the reduce, scan, MV and ragged-reduce
 * calls with CUDANP_MAP_AUTO / CUDANP_MAP_INTRA_WARP, and by TMV with the
 * inter-warp map for S = 64 / 128 (8 column-masters x S slave warps per CTA).
 * Teams larger than a CTA -- one thread-block cluster of 8 CTAs per item, the
 * CTAs' partials (and scan totals) meeting in shared memory over DSMEM, the
 * inter-warp smem exchange of P:203/P:209 one level up (np_cluster.cu), for
 * few outer items with very long loops:
 *   S in {2048, 4096, 8192}: batched reduce, batched scan and MV (S/8
 *     threads per CTA); CUDANP_ERR_INVALID for TMV;
 *   S in {256, 1024} with the inter-warp map: TMV (8 column-masters x 32 /
 *     128 slave warps per CTA).
 * Other (S, map) combinations return CUDANP_ERR_UNSUPPORTED.
 *
 * Conventions for every call:
 *  - Data pointers are DEVICE pointers owned by the caller; the library never
 *    allocates, frees or retains them.  Matrices and item arrays are
 *    row-major fp32/int32.  Outputs must not overlap inputs.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *    stream).  Calls validate their arguments synchronously, enqueue work on
 *    `stream` and return without synchronizing.  No C++ exception crosses
 *    the ABI.  The functions keep no state and are thread-safe.
 *  - Return value: a cudanp_status.  CUDANP_ERR_INVALID is returned before
 *    any launch (no partial work).  CUDANP_ERR_CUDA reports a launch error
 *    (text in cudanp_last_error()); faults during asynchronous execution
 *    surface at the caller's next synchronization.
 *  - N = 0 or L = 0 is valid: reduce writes init (or the identity) for each
 *    item, scan writes nothing, TMV/MV write 0 when the inner count is 0.
 *  - Misaligned pointers or leading dimensions that are not multiples of 4
 *    are not errors; they take the scalar (non-128-bit) path, except the
 *    intra-warp batched reduce, which peels each row to its 16-byte boundary
 *    and streams the rest in 128-bit units.
 */
#ifndef CUDANP_H_
#define CUDANP_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  CUDANP_OK = 0,
  CUDANP_ERR_INVALID = 1,     /* bad argument; nothing launched            */
  CUDANP_ERR_UNSUPPORTED = 2, /* valid but not built (e.g. intra-warp S=3) */
  CUDANP_ERR_CUDA = 3,        /* CUDA runtime error at launch              */
  CUDANP_ERR_NCCL = 4         /* reserved for collective errors            */
} cudanp_status;

typedef enum { CUDANP_DIST_CYCLIC = 0, CUDANP_DIST_BLOCK = 1 } cudanp_dist;
typedef enum {
  CUDANP_MAP_AUTO = 0,
  CUDANP_MAP_INTRA_WARP = 1,
  CUDANP_MAP_INTER_WARP = 2,
  CUDANP_MAP_INTER_WARP_TMA = 3, /* cudanp_tmv only: inter-warp, A staged by TMA (= cudanp_tmv_tma) */
  CUDANP_MAP_INTRA_WARP_TMA = 4  /* cudanp_batched_loop_reduce only: intra-warp teams fed from a
                                    TMA bulk-copy ring (= cudanp_batched_loop_reduce_tma) */
} cudanp_map;
typedef enum { CUDANP_F32 = 0, CUDANP_I32 = 1 } cudanp_dtype;
enum { CUDANP_S_AUTO = 0 }; /* S argument: the library picks the team size */
typedef enum { CUDANP_SUM = 0, CUDANP_MAX = 1 } cudanp_op;

/* ------------------------------------------------------------------------
 * The four hot-path calls (north star).
 * ---------------------------------------------------------------------- */

/* TMV, Fig 2: y[j] = sum_{i<n_inner} A[i*lda + j] * x[i], for
 * j < n_outer.  Master = column j (one output per master); the inner loop
 * runs over the h = n_inner rows.  A: n_inner x lda fp32 (lda >= n_outer),
 * x: n_inner fp32, y: n_outer fp32.  fp32 FMA accumulation; the S partial
 * sums are combined by the team reduction.  map = CUDANP_MAP_INTER_WARP_TMA
 * runs the TMA-staged kernel (cudanp_tmv_tma) when S is a power of two <= 32
 * and its preconditions hold, else the LDG inter-warp kernel (same result
 * contract; never CUDANP_ERR_UNSUPPORTED for alignment).  CUDANP_MAP_AUTO
 * takes the TMA-staged kernel under the same conditions when the 128-column
 * strips give 0.3 .. 1.1 CTAs per SM (one resident strip per SM with a deep
 * ring), else the LDG inter-warp kernel (adjacent
 * masters read adjacent columns). */
int cudanp_tmv(const float* A, int64_t lda, const float* x, float* y,
               int64_t n_outer, int64_t n_inner, int S, int dist, int map, void* stream);

/* TMV with TMA-staged tiles (north star: "TMA or cp.async staging where the
 * access pattern is strided (as in y=A^T x)"): the inter-warp map of
 * cudanp_tmv (Fig 2).  A CTA owns a strip of COLS
 * columns (32 column-masters x V) and S slave warps; a dedicated producer
 * warp (S <= 16; thread 0 for S = 32) streams [R rows x COLS] boxes of A
 * into a ring of shared-memory stages with cp.async.bulk.tensor (one
 * full/empty mbarrier pair per stage) and the slaves consume their rows,
 * cyclic or block (R5).  The shape makes the whole grid resident
 * at once.  Same result contract as cudanp_tmv (the S partial
 * sums meet in slave order).  Needs A 16-byte aligned, lda % 4 == 0 and both
 * sizes < 2^31 (TMA coordinates are int32), else CUDANP_ERR_UNSUPPORTED
 * (cudanp_tmv handles any case); x and y need no alignment (y is written
 * with scalar stores, so y may point into another buffer, e.g. a fused
 * gather's root + begin).  Columns past n_outer and rows past n_inner are
 * zero-filled by TMA and never stored; rows of a block-distribution box
 * that belong to the next slave are skipped, not multiplied by zero. */
int cudanp_tmv_tma(const float* A, int64_t lda, const float* x, float* y,
                   int64_t n_outer, int64_t n_inner, int S, int dist, void* stream);
/* Same with the launch shape pinned (tuning / the sweep): cols in {0 = auto,
 * 32, 64, 128} columns per CTA; rows_sel in {-1 = auto, 0, 1, 2} picks one
 * of three rows-per-slave-per-stage sizes for this S (each twice the last); stages 0 = auto,
 * else 2..64 ring stages (CUDANP_ERR_INVALID if the ring exceeds 227 KB). */
int cudanp_tmv_tma_ex(const float* A, int64_t lda, const float* x, float* y,
                      int64_t n_outer, int64_t n_inner, int S, int dist,
                      int cols, int rows_sel, int stages, void* stream);

/* MV (Table 1 "MV"): y[i] = sum_{j<n_inner} A[i*lda + j] * x[j],
 * for i < n_outer.  Master = row i; inner loop over the w = n_inner columns.
 * A: n_outer x lda fp32 (lda >= n_inner), x: n_inner, y: n_outer. */
int cudanp_mv(const float* A, int64_t lda, const float* x, float* y,
              int64_t n_outer, int64_t n_inner, int S, int dist, int map, void* stream);

/* Batched loop-reduce (reduction clause; Fig 6d):
 * out[n] = init[n] (op) fold_{i<L} in[n*L + i] for n < N = n_outer,
 * L = n_inner.  Item-major [N][L] layout.  dtype CUDANP_F32 or CUDANP_I32;
 * op CUDANP_SUM (int32 wraps modulo 2^32, R13) or CUDANP_MAX (identity -inf /
 * INT32_MIN, R14).  init may be NULL (identity).  The master loads init[n]
 * and stores out[n]. */
int cudanp_batched_loop_reduce(const void* in, const void* init, void* out,
                               int64_t n_outer, int64_t n_inner, int dtype, int op,
                               int S, int dist, int map, void* stream);

/* Team-reduction backend ablation (Fig 16: shfl vs shared
 * memory for the reduction under intra-warp NP; plus sm_100a redux.sync):
 * the batched loop-reduce with the intra-warp map and cyclic distribution,
 * combining the team's partials with backend 0 = shfl-xor butterfly (what
 * cudanp_batched_loop_reduce uses), 1 = shared memory (each lane writes a
 * slot, the master folds its team's S slots), 2 = redux.sync over the team's
 * lane mask (int32 add/max, fp32 max; fp32 sum -> CUDANP_ERR_UNSUPPORTED).
 * Built for the 128-bit path only: L % 4 == 0 and `in` 16-byte aligned, else
 * CUDANP_ERR_UNSUPPORTED. */
int cudanp_batched_loop_reduce_backend(const void* in, const void* init, void* out,
                                       int64_t n_outer, int64_t n_inner, int dtype, int op,
                                       int S, int backend, void* stream);

/* Batched loop-reduce with the loop body staged by TMA (same contract and
 * bit-identical results as cudanp_batched_loop_reduce with the intra-warp
 * map; map = CUDANP_MAP_INTRA_WARP_TMA there selects it): a producer warp
 * streams runs of consecutive items -- one contiguous block each -- into a
 * ring of shared-memory stages with cp.async.bulk, eight consumer warps run
 * the S-lane teams (S <= 32) out of shared memory.  stage_bytes (0 = 64 KB)
 * and stages (0 = as many as fit, <= 6) shape the ring.  Needs `in` 16-byte
 * aligned and n_inner % 4 == 0, else CUDANP_ERR_UNSUPPORTED. */
int cudanp_batched_loop_reduce_tma(const void* in, const void* init, void* out,
                                   int64_t n_outer, int64_t n_inner, int dtype, int op,
                                   int S, int dist, int stage_bytes, int stages, void* stream);

/* Batched inclusive scan (scan clause; inclusive per R1):
 * out[n*L + k] = init[n] + sum_{i<=k} in[n*L + i].  init may be NULL (0);
 * when given, the master loads it and broadcasts it to its slaves with
 * read_from_master.  Every team member stores its own elements. */
int cudanp_batched_loop_scan(const void* in, const void* init, void* out,
                             int64_t n_outer, int64_t n_inner, int dtype,
                             int S, int dist, int map, void* stream);

/* Ragged (runtime-bounded) loop-reduce over CSR segments (
 * P:193 "valid if the loop bound is determined at the runtime"):
 * out[n] = init[n] (op) fold_{offsets[n] <= i < offsets[n+1]} in[i], n < N.
 * offsets: N+1 int64 device values (8-byte aligned), non-decreasing; a
 * decreasing pair is treated as an empty loop.  The master of item n loads
 * its two bounds and broadcasts them with read_from_master;
 * the team streams the segment (head <= 3 scalars, 128-bit aligned body,
 * tail <= 3 scalars).  in and offsets must be non-NULL when N > 0.  dtype,
 * op, init, S, dist, map as for cudanp_batched_loop_reduce. */
int cudanp_ragged_loop_reduce(const void* in, const int64_t* offsets, const void* init, void* out,
                              int64_t n_outer, int dtype, int op, int S, int dist, int map,
                              void* stream);
/* Ragged reduce with the team size chosen per segment at run time: each lane
 * of a warp is the master of one segment; segments shorter than `threshold`
 * elements are reduced by their master alone (S = 1, 128-bit body units),
 * longer ones by the whole warp as a team of 32 (cyclic units, shfl
 * reduction), the masters taking turns -- the master decides in its
 * sequential section whether to wake its slaves for a loop whose bound it has
 * just read (the imbalance of P:340 under length mixes).  Same
 * result contract as cudanp_ragged_loop_reduce; threshold >= 1, else
 * CUDANP_ERR_INVALID. */
int cudanp_ragged_loop_reduce_adaptive(const void* in, const int64_t* offsets, const void* init,
                                       void* out, int64_t n_outer, int dtype, int op,
                                       int64_t threshold, void* stream);
/* Comparison: one thread per segment, serial loop (Fig 2 style). */
int cudanp_ragged_loop_reduce_literal(const void* in, const int64_t* offsets, const void* init,
                                      void* out, int64_t n_outer, int dtype, int op, void* stream);

/* Multi-section items, the LE kernel of Figs 5-6 (SURVEY §8(f)
 * f2): per item n with L = n_inner points Grad[i] = in(n, i):
 *   sum = reduction(Grad); ave = sum / L;
 *   var = reduction((Grad-ave)^2); ep = reduction(Grad-ave);
 *   if ((ave*ave)/var > threshold) gicov[n] = ave / sqrt(var)   (master only)
 * gicov[n] is left untouched when the test fails.  ave, var,
 * ep (N floats each) may be NULL.  layout 0: in[n*L + i] (item-major);
 * layout 1: in[i*N + n] (point-major).  Grad stays in the slaves' registers
 * between the loops (Fig 6c) when ceil(L/S) <= 32.  S: 1,2,4,8,16,32 for
 * both maps, and also 3,5,10,15 for CUDANP_MAP_INTER_WARP (Fig 12);
 * a non-power-of-two S with the intra-warp map returns
 * CUDANP_ERR_UNSUPPORTED.  L must be >= 1 when N > 0. */
int cudanp_le_gicov(const float* in, float* gicov, float* ave, float* var, float* ep,
                    int64_t n_outer, int64_t n_inner, float threshold, int layout, int S,
                    int dist, int map, void* stream);
/* The same with the home of Grad chosen (Fig 6a-c; Fig 15):
 * CUDANP_GRAD_REGISTERS = cudanp_le_gicov (6c, per-slave register partition);
 * CUDANP_GRAD_GLOBAL (6a: no private copy, loop 3 re-reads the input through
 * L1/L2); CUDANP_GRAD_SHARED (6b: runs of whole items are staged in a
 * shared-memory ring by TMA bulk copies and both loops read it there; built
 * for layout 0, the intra-warp map, S = 2^k <= 32 and a 16-byte aligned
 * input, else CUDANP_ERR_UNSUPPORTED; the < 4 items past the last whole
 * 16-byte run take the register kernel).  All three give
 * bit-identical results (each slave visits its elements in the same order). */
typedef enum { CUDANP_GRAD_REGISTERS = 0, CUDANP_GRAD_SHARED = 1, CUDANP_GRAD_GLOBAL = 2 } cudanp_grad_placement;
int cudanp_le_gicov_placement(const float* in, float* gicov, float* ave, float* var, float* ep,
                              int64_t n_outer, int64_t n_inner, float threshold, int layout,
                              int S, int dist, int map, int placement, void* stream);
/* Comparison: Fig 5 as written, one thread per item, Grad in a per-thread
 * local-memory array when L <= 256. */
int cudanp_le_gicov_literal(const float* in, float* gicov, float* ave, float* var, float* ep,
                            int64_t n_outer, int64_t n_inner, float threshold, int layout,
                            void* stream);

/* ------------------------------------------------------------------------
 * Comparison kernels.  Same operands as the NP
 * call; `impl` selects:
 *   CUDANP_IMPL_S1_LITERAL: Fig 2 verbatim -- one thread per item, scalar
 *       serial loop, no vector loads;
 *   CUDANP_IMPL_DP_THREAD : CUDA dynamic parallelism (CDP2): every master
 *       launches a child grid for its loop; the child stores the result;
 *   CUDANP_IMPL_DP_BLOCK  : DP with one child launch per thread block (the
 *       paper's manual optimisation);
 *   CUDANP_IMPL_S1_TILED  : the tuned no-NP baseline -- one thread per item
 *       (S = 1) whose rows reach it through shared-memory tiles copied by TMA
 *       (the "already optimized" SMM-style baseline of P:411 / Table 1):
 *       MV, reduce and scan (np_s1_tiled.cu; scan tiles are stored back by
 *       TMA), TMV (= cudanp_tmv_tma with S = 1).  Needs 16-byte aligned operands with rows a multiple of
 *       4 elements (and sizes < 2^31), else CUDANP_ERR_UNSUPPORTED.
 * DP variants need enough device-runtime launch slots: see
 * cudanp_dp_set_pending_launch_limit.  A DP launch that the device runtime
 * refuses sets a device error flag; cudanp_dp_error_count() reads it.
 * ---------------------------------------------------------------------- */
typedef enum {
  CUDANP_IMPL_S1_LITERAL = 1,
  CUDANP_IMPL_DP_THREAD = 2,
  CUDANP_IMPL_DP_BLOCK = 3,
  CUDANP_IMPL_S1_TILED = 4
} cudanp_impl;

int cudanp_tmv_variant(int impl, const float* A, int64_t lda, const float* x, float* y,
                       int64_t n_outer, int64_t n_inner, void* stream);
int cudanp_mv_variant(int impl, const float* A, int64_t lda, const float* x, float* y,
                      int64_t n_outer, int64_t n_inner, void* stream);
int cudanp_batched_loop_reduce_variant(int impl, const void* in, const void* init, void* out,
                                       int64_t n_outer, int64_t n_inner, int dtype, int op,
                                       void* stream);
int cudanp_batched_loop_scan_variant(int impl, const void* in, const void* init, void* out,
                                     int64_t n_outer, int64_t n_inner, int dtype, void* stream);
/* cudaDeviceSetLimit(cudaLimitDevRuntimePendingLaunchCount, n) on the
 * current device. */
int cudanp_dp_set_pending_launch_limit(size_t n);
/* Number of device-side child launches that failed since the last reset
 * (synchronizes the device); reset = 1 clears the counter. */
int cudanp_dp_error_count(int reset, int64_t* count_out);

/* Memory-copy microbenchmark of Fig 1: copies
 * `total` floats in -> out.  variant 0: plain grid-stride copy kernel built
 * without relocatable device code; 1: the same kernel built with -rdc (the
 * "dynamic-parallelism-enabled kernel overhead"); 2: dynamic
 * parallelism -- a parent kernel of m threads, each launching a child grid
 * of n = total/m threads that copies n floats (m must divide total). */
int cudanp_dp_memcopy(const float* in, float* out, int64_t total, int64_t m, int variant,
                      void* stream);

/* ------------------------------------------------------------------------
 * Version selection (the paper's exhaustive autotune, P:384, P:413,
 * P:484-486): op_kind 0 tmv, 1 mv, 2 reduce, 3 scan.  The candidates are the
 * library's (S, dist, map) instantiations (S = 1..32 x cyclic/block x
 * intra/inter, plus multi-warp teams); cudanp_autotune_count/_candidate list
 * them.  cudanp_autotune runs each candidate once as warm-up and `reps` times
 * under CUDA events on `stream` with the caller's operands (a = A or in,
 * b = x or init, out = y or out; lda for tmv/mv; dtype/op for reduce, dtype
 * for scan), writes the mean ms per launch to ms_table[i] (INFINITY for a
 * combination this shape does not support, and for a team larger than both
 * a warp and the loop -- S > 32 and S > n_inner: slaves without a single
 * iteration, not timed; ms_table may be NULL) and the
 * fastest candidate's index to *best_index.  Synchronizes `stream`.  `out` is
 * overwritten by every candidate (the last run's result is valid). */
int cudanp_autotune_count(int op_kind);
int cudanp_autotune_candidate(int op_kind, int index, int* S, int* dist, int* map);
int cudanp_autotune(int op_kind, const void* a, const void* b, void* out, int64_t lda,
                    int64_t n_outer, int64_t n_inner, int dtype, int op, int reps,
                    float* ms_table, int* best_index, void* stream);

/* ------------------------------------------------------------------------
 * Launch shape actually used (the paper's resource analysis, Table 1 P:96,
 * and autotune space P:384): for an NP call with these arguments,
 * report the kernel's block size, grid size, registers per thread, static
 * shared memory bytes and the resolved map.  `op_kind`: 0 tmv, 1 mv,
 * 2 reduce, 3 scan, 4 TMA-staged tmv, 5 TMA-staged reduce (dynamic shared
 * memory of their rings in smem_bytes).  vec4 != 0 states that the operands
 * are 16-byte aligned with rows a multiple of 4 elements (the 128-bit and TMA
 * paths).  S = CUDANP_S_AUTO and MAP_AUTO resolve as in the calls; the
 * resolved map (CUDANP_MAP_INTER_WARP_TMA when TMV takes the TMA kernel), S
 * and dist are returned.  Any out pointer may be NULL.
 * ---------------------------------------------------------------------- */
int cudanp_launch_info(int op_kind, int64_t n_outer, int64_t n_inner, int dtype, int op,
                       int S, int dist, int map, int vec4,
                       int* block_threads, int64_t* grid_ctas, int* regs_per_thread,
                       int* smem_bytes, int* resolved_map, int* S_used, int* dist_used);

/* The (S, dist, map) that S = CUDANP_S_AUTO selects for op_kind (0 tmv, 1 mv,
 * 2 reduce, 3 scan) on N = n_outer items of L = n_inner iterations, given
 * `map` (AUTO, or a map to keep) and vec4 as above.  Rule:
 * TMV with 0.3..1.1 128-column strips per SM -> TMA S = 8 cyclic (with vec4
 * only from 0.75 strips per SM, below that the S = 128 inter rule); wider ->
 * inter-warp S = 32 block; narrower -> inter-warp S = 128 with vec4 (else
 * clamp(2*SMs*1024/N, 8, 64)), block when L/S < 32 (and N > 1024 with
 * vec4), else cyclic;
 * MV intra S = clamp(L/64, 1, 256); reduce intra S = clamp(L/8, 1, 32);
 * scan intra S = clamp(L/4, 1, 16); reduce/scan/MV teams grow (up to S/32
 * warps, slaves keeping >= 8 elements) while N*S < SMs*1024. */
int cudanp_choose_version(int op_kind, int64_t n_outer, int64_t n_inner, int vec4, int map,
                          int* S, int* dist, int* map_out);

/* ------------------------------------------------------------------------
 * Multi-GPU helper (one process per GPU; outer items are independent,
 * P:13): the contiguous range [floor(g*N/G), floor((g+1)*N/G)) that
 * rank g of G owns.
 * ---------------------------------------------------------------------- */
int cudanp_shard_range(int64_t n_outer, int nranks, int rank, int64_t* begin, int64_t* end);

/* Native multi-GPU group, one process per GPU: a group is
 * this process's rank of an NCCL communicator on the current device.
 * cudanp_group_unique_id: rank 0 writes 128 opaque bytes to id_out, which the
 *   caller hands to every rank (any channel).
 * cudanp_group_create: every rank, with the same id, nranks and its rank
 *   (collective: blocks until all ranks joined).  *out is owned by the caller
 *   and released with cudanp_group_destroy.
 * cudanp_group_gather: the contiguous shard [begin_g, end_g) of n_total items
 *   (cudanp_shard_range) of every rank lands in root_buf on rank 0 (root_buf
 *   may be NULL elsewhere); NCCL send/recv enqueued on `stream`.
 * cudanp_sharded_tmv / cudanp_sharded_batched_loop_reduce: this rank's shard
 *   of the outer items (A_shard = the h x (end-begin) column block, lda its row
 *   stride, x all h rows; in_shard = items [begin, end)) through the NP call,
 *   then the gather to y_root / out_root on rank 0.  Same argument rules as
 *   the single-GPU calls.
 * NCCL is loaded at run time (libnccl.so.2); CUDANP_ERR_NCCL if it cannot be,
 * or on any NCCL failure (text in cudanp_last_error()). */
typedef struct cudanp_group cudanp_group;
int cudanp_group_unique_id(void* id_out);
int cudanp_group_create(const void* id, int nranks, int rank, cudanp_group** out);
int cudanp_group_destroy(cudanp_group* group);
int cudanp_group_rank(const cudanp_group* group, int* rank, int* nranks);
int cudanp_group_gather(cudanp_group* group, const void* local, void* root_buf, int64_t n_total,
                        int dtype, void* stream);
int cudanp_sharded_tmv(cudanp_group* group, const float* A_shard, int64_t lda, const float* x,
                       float* y_shard, float* y_root, int64_t n_outer_total, int64_t n_inner,
                       int S, int dist, int map, void* stream);
int cudanp_sharded_batched_loop_reduce(cudanp_group* group, const void* in_shard,
                                       const void* init_shard, void* out_shard, void* out_root,
                                       int64_t n_outer_total, int64_t n_inner, int dtype, int op,
                                       int S, int dist, int map, void* stream);

/* Fused gather over NVLink: CUDA IPC lets rank g's kernel
 * epilogue store its outputs straight into rank 0's result buffer, so the
 * master's store *is* the gather -- pass the opened pointer (plus the
 * shard's begin) as the `y`/`out` argument of any call above.
 * cudanp_ipc_get_handle: handle_out receives 64 bytes (cudaIpcMemHandle_t) of
 *   the allocation holding dev_ptr and *offset_out its byte offset in it.
 * cudanp_ipc_open: maps a handle from another process of the same node;
 *   *dev_ptr_out = mapped base + offset.  Peer access is enabled lazily.
 * cudanp_ipc_close: unmaps (pass the pointer and offset from ipc_open).
 * The caller orders the writes (stream sync + a barrier) before the owner
 * reads the buffer. */
int cudanp_ipc_get_handle(const void* dev_ptr, void* handle_out, int64_t* offset_out);
int cudanp_ipc_open(const void* handle, int64_t offset, void** dev_ptr_out);
int cudanp_ipc_close(void* dev_ptr, int64_t offset);

/* ------------------------------------------------------------------------
 * Test and benchmark support (not part of the method).
 * ---------------------------------------------------------------------- */

/* Device-side counter-based input generator:
 * out[r*ld + c] = value(kind, splitmix64(splitmix64(seed ^ (stream_id<<56))
 * ^ ((row0 + r) * w_global + col0 + c))) for r < rows, c < cols.
 * kind: 0 f32_unit, 1 f32_signed, 2 f32_int4, 3 i32_small (parameter B),
 * 4 i32_full, 5 ones (fp32), 6 ones (int32).  B must be a power of two. */
int cudanp_generate(void* out, int64_t rows, int64_t cols, int64_t ld, int64_t row0,
                    int64_t col0, int64_t w_global, int stream_id, int kind, int64_t B,
                    uint64_t seed, void* stream);

/* Runs the kernels' own iteration-distribution code on the device and copies
 * owner[u*V + k] = slave that executes element u*V+k of a loop of n_inner
 * elements back to the HOST array owner_host (n_inner int32).  V in {1,4}.
 * Synchronous. */
int cudanp_debug_owner_map(int64_t n_inner, int S, int dist, int V, int32_t* owner_host);

/* Runs the kernels' own team formation for one CTA of `map` with team size S
 * on the device and copies master/slave ids of each linear thread id to the
 * HOST arrays (nthreads = 32*S for inter-warp, 32 for intra-warp).
 * Synchronous.  Returns the thread count through *nthreads. */
int cudanp_debug_team_ids(int S, int map, int32_t* master_host, int32_t* slave_host,
                          int* nthreads);

/* Runs read_from_master on the device: for each team of a warp (intra) or
 * CTA (inter), every member returns the value its master held; values[t] =
 * 1000*t + 7 before, out_host[t] after.  Synchronous. */
int cudanp_debug_broadcast(int S, int map, int32_t* out_host, int* nthreads);

const char* cudanp_status_string(int status);
/* Detail text for the last non-OK return on this host thread. */
const char* cudanp_last_error(void);
/* Library version as major*10000 + minor*100 + patch. */
int cudanp_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CUDANP_H_ */
