/* abi_client.c -- a plain C99 client of libcudanp.so: the boundary used
 * without Python or torch (include/cudanp.h + the CUDA runtime only).
 *
 * It allocates device memory itself, calls the four hot-path entry points on
 * a stream it created, and checks closed forms that hold for any correct
 * implementation (SURVEY C-3 pin P2; north star: "A=all-ones giving y_j =
 * sum of x; a scan of ones giving 1..L"):
 *   TMV with A = all ones        -> y[j] = sum_i x[i]       (Fig 2)
 *   MV  with A = all ones        -> y[i] = sum_j x[j]
 *   reduce of ones (int32, sum)  -> L; of 0..L-1 (max) -> L-1
 *   scan of ones (int32)         -> 1..L
 * with small-integer x so every fp32 sum is exact -- for S = CUDANP_S_AUTO
 * (the library's choice), S = 1, 4, 32, 256 and the inter-warp-only S = 5,
 * and for the TMA-tiled S=1 baselines (CUDANP_IMPL_S1_TILED).  It also checks
 * that a bad argument is rejected before any launch with CUDANP_ERR_INVALID
 * and an unbuilt combination with CUDANP_ERR_UNSUPPORTED.
 * Exit code 0 = all checks passed.  Test infrastructure, not product code. */
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <cuda_runtime.h>

#include "cudanp.h"

#define CK(x)                                                                      \
  do {                                                                             \
    cudaError_t e_ = (x);                                                          \
    if (e_ != cudaSuccess) {                                                       \
      fprintf(stderr, "%s:%d CUDA: %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); \
      return 2;                                                                    \
    }                                                                              \
  } while (0)
#define NP(x)                                                                      \
  do {                                                                             \
    int s_ = (x);                                                                  \
    if (s_ != CUDANP_OK) {                                                         \
      fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, cudanp_status_string(s_), \
              cudanp_last_error());                                                \
      return 3;                                                                    \
    }                                                                              \
  } while (0)

int main(void) {
  const int64_t h = 777, w = 1030, N = 5000, L = 150;
  const int Ss[] = {CUDANP_S_AUTO, 1, 4, 5, 32, 256};
  int fails = 0;
  cudaStream_t st;
  CK(cudaStreamCreate(&st));

  float *A, *x, *y, *hx, *hy;
  int32_t *in, *out, *hin, *hout;
  CK(cudaMalloc((void**)&A, sizeof(float) * h * w));
  CK(cudaMalloc((void**)&x, sizeof(float) * (h > w ? h : w)));
  CK(cudaMalloc((void**)&y, sizeof(float) * (h > w ? h : w)));
  CK(cudaMalloc((void**)&in, sizeof(int32_t) * N * L));
  CK(cudaMalloc((void**)&out, sizeof(int32_t) * N * L));
  hx = (float*)malloc(sizeof(float) * (h > w ? h : w));
  hy = (float*)malloc(sizeof(float) * (h > w ? h : w));
  hin = (int32_t*)malloc(sizeof(int32_t) * N * L);
  hout = (int32_t*)malloc(sizeof(int32_t) * N * L);

  float* ones = (float*)malloc(sizeof(float) * h * w);
  for (int64_t i = 0; i < h * w; ++i) ones[i] = 1.0f;
  CK(cudaMemcpy(A, ones, sizeof(float) * h * w, cudaMemcpyHostToDevice));
  free(ones);
  for (int64_t i = 0; i < (h > w ? h : w); ++i) hx[i] = (float)(i % 7);
  CK(cudaMemcpy(x, hx, sizeof(float) * (h > w ? h : w), cudaMemcpyHostToDevice));

  for (int k = 0; k < 6; ++k) {
    for (int dist = 0; dist < 2; ++dist) {
      const int S = Ss[k];
      /* TMV: y[j] = sum_{i<h} x[i] */
      double sx = 0;
      for (int64_t i = 0; i < h; ++i) sx += hx[i];
      if (S <= 128) {
        NP(cudanp_tmv(A, w, x, y, w, h, S, dist, CUDANP_MAP_AUTO, st));
        CK(cudaMemcpyAsync(hy, y, sizeof(float) * w, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        for (int64_t j = 0; j < w; ++j)
          if (hy[j] != (float)sx) { fprintf(stderr, "tmv S=%d j=%ld: %g != %g\n", S, (long)j, hy[j], sx); ++fails; break; }
      }
      /* MV: y[i] = sum_{j<w} x[j] */
      sx = 0;
      for (int64_t j = 0; j < w; ++j) sx += hx[j];
      NP(cudanp_mv(A, w, x, y, h, w, S, dist, CUDANP_MAP_AUTO, st));
      CK(cudaMemcpyAsync(hy, y, sizeof(float) * h, cudaMemcpyDeviceToHost, st));
      CK(cudaStreamSynchronize(st));
      for (int64_t i = 0; i < h; ++i)
        if (hy[i] != (float)sx) { fprintf(stderr, "mv S=%d i=%ld: %g != %g\n", S, (long)i, hy[i], sx); ++fails; break; }

      /* reduce of ones -> L; max of 0..L-1 -> L-1; scan of ones -> 1..L */
      for (int64_t i = 0; i < N * L; ++i) hin[i] = 1;
      CK(cudaMemcpy(in, hin, sizeof(int32_t) * N * L, cudaMemcpyHostToDevice));
      NP(cudanp_batched_loop_reduce(in, NULL, out, N, L, CUDANP_I32, CUDANP_SUM, S, dist, CUDANP_MAP_AUTO, st));
      CK(cudaMemcpyAsync(hout, out, sizeof(int32_t) * N, cudaMemcpyDeviceToHost, st));
      CK(cudaStreamSynchronize(st));
      for (int64_t n = 0; n < N; ++n)
        if (hout[n] != L) { fprintf(stderr, "reduce S=%d n=%ld: %d\n", S, (long)n, hout[n]); ++fails; break; }
      NP(cudanp_batched_loop_scan(in, NULL, out, N, L, CUDANP_I32, S, dist, CUDANP_MAP_AUTO, st));
      CK(cudaMemcpyAsync(hout, out, sizeof(int32_t) * N * L, cudaMemcpyDeviceToHost, st));
      CK(cudaStreamSynchronize(st));
      for (int64_t i = 0; i < N * L; ++i)
        if (hout[i] != (int32_t)(i % L) + 1) { fprintf(stderr, "scan S=%d i=%ld: %d\n", S, (long)i, hout[i]); ++fails; break; }
      for (int64_t i = 0; i < N * L; ++i) hin[i] = (int32_t)((i * 7919) % L);  /* a permutation of 0..L-1 per row (gcd(7919,150)=1) */
      CK(cudaMemcpy(in, hin, sizeof(int32_t) * N * L, cudaMemcpyHostToDevice));
      NP(cudanp_batched_loop_reduce(in, NULL, out, N, L, CUDANP_I32, CUDANP_MAX, S, dist, CUDANP_MAP_AUTO, st));
      CK(cudaMemcpyAsync(hout, out, sizeof(int32_t) * N, cudaMemcpyDeviceToHost, st));
      CK(cudaStreamSynchronize(st));
      for (int64_t n = 0; n < N; ++n)
        if (hout[n] != L - 1) { fprintf(stderr, "max S=%d n=%ld: %d\n", S, (long)n, hout[n]); ++fails; break; }
    }
  }
  /* tiled S=1 baselines on rows of 148 elements (a multiple of 4): scan of ones -> 1..148,
   * reduce of ones -> 148 */
  {
    const int64_t L4 = 148;
    for (int64_t i = 0; i < N * L4; ++i) hin[i] = 1;
    CK(cudaMemcpy(in, hin, sizeof(int32_t) * N * L4, cudaMemcpyHostToDevice));
    NP(cudanp_batched_loop_scan_variant(CUDANP_IMPL_S1_TILED, in, NULL, out, N, L4, CUDANP_I32, st));
    CK(cudaMemcpyAsync(hout, out, sizeof(int32_t) * N * L4, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    for (int64_t i = 0; i < N * L4; ++i)
      if (hout[i] != (int32_t)(i % L4) + 1) { fprintf(stderr, "tiled scan i=%ld: %d\n", (long)i, hout[i]); ++fails; break; }
    NP(cudanp_batched_loop_reduce_variant(CUDANP_IMPL_S1_TILED, in, NULL, out, N, L4, CUDANP_I32, CUDANP_SUM, st));
    CK(cudaMemcpyAsync(hout, out, sizeof(int32_t) * N, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    for (int64_t n = 0; n < N; ++n)
      if (hout[n] != L4) { fprintf(stderr, "tiled reduce n=%ld: %d\n", (long)n, hout[n]); ++fails; break; }
    /* rows of 150 elements cannot be described to TMA: unsupported, not wrong */
    if (cudanp_batched_loop_scan_variant(CUDANP_IMPL_S1_TILED, in, NULL, out, N, L, CUDANP_I32, st) !=
        CUDANP_ERR_UNSUPPORTED) {
      fprintf(stderr, "tiled scan with L %% 4 != 0 was not refused\n");
      ++fails;
    }
  }
  /* intra-warp teams need S = 2^k: S = 5 intra-warp is unsupported */
  if (cudanp_batched_loop_reduce(in, NULL, out, N, L, CUDANP_I32, CUDANP_SUM, 5, 0, CUDANP_MAP_INTRA_WARP, st) !=
      CUDANP_ERR_UNSUPPORTED) {
    fprintf(stderr, "S=5 intra-warp was not refused\n");
    ++fails;
  }
  /* validation before launch: S = 6 is not a team size (3, 5, 10, 15 are, inter-warp) */
  if (cudanp_batched_loop_reduce(in, NULL, out, N, L, CUDANP_I32, CUDANP_SUM, 6, 0, 0, st) != CUDANP_ERR_INVALID) {
    fprintf(stderr, "S=6 was not rejected\n");
    ++fails;
  }
  CK(cudaStreamSynchronize(st));
  printf("abi_client: %s (%d failures), libcudanp version %d\n", fails ? "FAIL" : "OK", fails, cudanp_version());
  cudaFree(A); cudaFree(x); cudaFree(y); cudaFree(in); cudaFree(out);
  free(hx); free(hy); free(hin); free(hout);
  cudaStreamDestroy(st);
  return fails ? 1 : 0;
}
