/* host_stream.c -- host DRAM bandwidth on the GPU box (OpenMP copy and a
 * 5-read/4-write pattern like the host-compute AdamW), for the HOST_COMPUTE
 * roofline.  gcc -O3 -march=native -fopenmp -o build/host_stream tools/host_stream.c */
#include <omp.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

static double now(void) { return omp_get_wtime(); }

int main(void) {
  const size_t n = (size_t)1 << 28;  /* 268M floats = 1 GiB per array */
  float *a = aligned_alloc(64, n * 4), *b = aligned_alloc(64, n * 4), *c = aligned_alloc(64, n * 4);
  uint16_t *g = aligned_alloc(64, n * 2), *p = aligned_alloc(64, n * 2);
#pragma omp parallel for
  for (size_t i = 0; i < n; ++i) { a[i] = 1.f; b[i] = 2.f; c[i] = 3.f; g[i] = 1; p[i] = 0; }
  double best_copy = 1e30, best_pat = 1e30;
  for (int r = 0; r < 5; ++r) {
    double t0 = now();
#pragma omp parallel for
    for (size_t i = 0; i < n; ++i) b[i] = a[i];
    double t1 = now();
    if (t1 - t0 < best_copy) best_copy = t1 - t0;
    t0 = now();
#pragma omp parallel for
    for (size_t i = 0; i < n; ++i) {
      float x = a[i] + (float)g[i], y = b[i] * 0.9f, z = c[i] * 0.99f;
      a[i] = x; b[i] = y; c[i] = z; p[i] = (uint16_t)i;
    }
    t1 = now();
    if (t1 - t0 < best_pat) best_pat = t1 - t0;
  }
  printf("{\"threads\": %d, \"copy_gbs\": %.1f, \"adam_pattern_gbs\": %.1f, \"adam_pattern_gparams\": %.2f}\n",
         omp_get_max_threads(), 8.0 * n / best_copy / 1e9, 28.0 * n / best_pat / 1e9, n / best_pat / 1e9);
  return 0;
}
