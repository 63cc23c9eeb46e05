// autotune.cu -- the paper's version selection, as a library call.
//
// CUDA-NP's compiler "generates multiple versions to explore different numbers
// of slave threads, and different thread distribution approaches" and picks
// the fastest by running them, since "CUDA-NP only generates a small number of
// versions, the optimal version can be found by testing these versions
// exhaustively".  Here the versions are the
// library's (S, dist, map) instantiations (for TMV also the TMA-staged
// inter-warp kernel, map CUDANP_MAP_INTER_WARP_TMA, and for reduce the
// TMA-staged intra-warp kernel, CUDANP_MAP_INTRA_WARP_TMA); cudanp_autotune times each one on
// the caller's operands with CUDA events on the caller's stream and reports
// the fastest.  Host code only: it calls the public entry points.
#include <cmath>
#include <vector>

#include "common.cuh"

namespace cudanp {

struct Candidate { int S, dist, map; };

static std::vector<Candidate> candidates(int op_kind) {
  std::vector<Candidate> c;
  const int small[] = {1, 2, 4, 8, 16, 32};
  for (int S : small)
    for (int d = 0; d < 2; ++d)
      for (int m = CUDANP_MAP_INTRA_WARP; m <= CUDANP_MAP_INTER_WARP; ++m) c.push_back({S, d, m});
  for (int S : {3, 5, 10, 15})  // non-power-of-two inter-warp teams (Fig 12)
    for (int d = 0; d < 2; ++d) c.push_back({S, d, CUDANP_MAP_INTER_WARP});
  if (op_kind == 0) {  // TMV: TMA-staged inter-warp, and inter-warp teams up to 128
    for (int S : small)
      for (int d = 0; d < 2; ++d) c.push_back({S, d, CUDANP_MAP_INTER_WARP_TMA});
    for (int S : {64, 128, 256, 1024})  // 256 / 1024: a cluster of 8 CTAs per column group
      for (int d = 0; d < 2; ++d) c.push_back({S, d, CUDANP_MAP_INTER_WARP});
  } else {             // MV / reduce / scan: multi-warp teams (+ the TMA-staged reduce, cluster teams)
    if (op_kind == 2)
      for (int S : small)
        for (int d = 0; d < 2; ++d) c.push_back({S, d, CUDANP_MAP_INTRA_WARP_TMA});
    for (int S : {64, 128, 256, 512, 1024})
      for (int d = 0; d < 2; ++d) c.push_back({S, d, CUDANP_MAP_INTRA_WARP});
    for (int S : {2048, 4096, 8192})  // cluster teams
      for (int d = 0; d < 2; ++d) c.push_back({S, d, CUDANP_MAP_INTRA_WARP});
  }
  return c;
}

static int run_one(int op_kind, const Candidate& k, const void* a, const void* b, void* out,
                   int64_t lda, int64_t N, int64_t L, int dtype, int op, void* stream) {
  switch (op_kind) {
    case 0: return cudanp_tmv((const float*)a, lda, (const float*)b, (float*)out, N, L, k.S, k.dist, k.map, stream);
    case 1: return cudanp_mv((const float*)a, lda, (const float*)b, (float*)out, N, L, k.S, k.dist, k.map, stream);
    case 2: return cudanp_batched_loop_reduce(a, b, out, N, L, dtype, op, k.S, k.dist, k.map, stream);
    case 3: return cudanp_batched_loop_scan(a, b, out, N, L, dtype, k.S, k.dist, k.map, stream);
    default: return fail_invalid("op_kind");
  }
}

}  // namespace cudanp

using namespace cudanp;

extern "C" {

int cudanp_autotune_count(int op_kind) {
  if (op_kind < 0 || op_kind > 3) return -1;
  return (int)candidates(op_kind).size();
}

int cudanp_autotune_candidate(int op_kind, int index, int* S, int* dist, int* map) {
  if (op_kind < 0 || op_kind > 3) return fail_invalid("op_kind");
  const auto c = candidates(op_kind);
  if (index < 0 || index >= (int)c.size() || !S || !dist || !map) return fail_invalid("candidate index");
  *S = c[index].S;
  *dist = c[index].dist;
  *map = c[index].map;
  return CUDANP_OK;
}

int cudanp_autotune(int op_kind, const void* a, const void* b, void* out, int64_t lda,
                    int64_t n_outer, int64_t n_inner, int dtype, int op, int reps,
                    float* ms_table, int* best_index, void* stream) {
  if (op_kind < 0 || op_kind > 3) return fail_invalid("op_kind");
  if (reps < 1) return fail_invalid("reps must be >= 1");
  if (!best_index) return fail_invalid("best_index is NULL");
  const auto c = candidates(op_kind);
  cudaStream_t st = (cudaStream_t)stream;
  cudaEvent_t e0, e1;
  if (cudaEventCreate(&e0) != cudaSuccess || cudaEventCreate(&e1) != cudaSuccess)
    return check_launch("cudaEventCreate");
  int best = -1;
  float best_ms = INFINITY;
  int rc = CUDANP_OK;
  for (size_t i = 0; i < c.size(); ++i) {
    float ms = INFINITY;
    if (c[i].S > 32 && c[i].S > n_inner) {
      // a team larger than both a warp and the loop: slaves without a single
      // iteration (P:426's idle slaves taken to the extreme) -- not a version
      // worth timing (C5's 64-element items under 8192-thread cluster teams
      // took ~6 s per launch)
      if (ms_table) ms_table[i] = ms;
      continue;
    }
    // warm-up launch doubles as the validity check (unsupported combos are skipped)
    int r = run_one(op_kind, c[i], a, b, out, lda, n_outer, n_inner, dtype, op, stream);
    if (r == CUDANP_OK) {
      cudaEventRecord(e0, st);
      for (int k = 0; k < reps && r == CUDANP_OK; ++k)
        r = run_one(op_kind, c[i], a, b, out, lda, n_outer, n_inner, dtype, op, stream);
      cudaEventRecord(e1, st);
      if (cudaEventSynchronize(e1) != cudaSuccess) { rc = check_launch("autotune sync"); break; }
      if (r == CUDANP_OK) {
        cudaEventElapsedTime(&ms, e0, e1);
        ms /= reps;
      }
    } else if (r == CUDANP_ERR_CUDA) {
      // A launch that the device refused (a configuration this device cannot
      // run) skips the candidate; a device that faulted ends the search.
      if (cudaStreamSynchronize(st) != cudaSuccess || cudaGetLastError() != cudaSuccess) {
        rc = check_launch("autotune: device error after a candidate");
        if (!rc) rc = CUDANP_ERR_CUDA;
        break;
      }
    }
    if (ms_table) ms_table[i] = ms;
    if (ms < best_ms) { best_ms = ms; best = (int)i; }
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  if (rc) return rc;
  if (best < 0) return fail_invalid("no candidate ran (check the operands)");
  *best_index = best;
  return CUDANP_OK;
}

}  // extern "C"
