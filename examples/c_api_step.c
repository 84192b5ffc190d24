/* c_api_step.c -- the C ABI used from plain C (no Python, no torch).
 *
 * One 1M-parameter block, device-resident: allocate P16/G16/P32/m/v with the
 * CUDA runtime, fill them with the library's seeded generator, arm three AGO
 * steps and hand the block off from a "backward" stream, sync, and print a
 * few updated values plus a P16 == bf16(P32) check.
 *
 * Build (from the repo root):
 *   nvcc -o build/c_api_step examples/c_api_step.c -Iinclude \
 *        -Lpaper_conf_icde_liaosyxcyww25_b200 -lratel \
 *        -Xlinker -rpath=$PWD/paper_conf_icde_liaosyxcyww25_b200
 */
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "ratel.h"
#include "ratel_gen.h"

#define CHECK(x)                                                                 \
  do {                                                                           \
    int rc_ = (x);                                                               \
    if (rc_ != RATEL_OK) {                                                       \
      fprintf(stderr, "%s -> %d: %s\n", #x, rc_, ratel_last_error());            \
      return 1;                                                                  \
    }                                                                            \
  } while (0)

int main(void) {
  const uint64_t n = 1000003; /* ragged on purpose */
  const uint64_t cap = ratel_padded_numel(n, 1);
  void *p16, *g16;
  float *theta, *m, *v;
  if (cudaMalloc(&p16, cap * 2) || cudaMalloc(&g16, cap * 2) || cudaMalloc((void**)&theta, n * 4) ||
      cudaMalloc((void**)&m, n * 4) || cudaMalloc((void**)&v, n * 4)) {
    fprintf(stderr, "cudaMalloc failed\n");
    return 1;
  }
  cudaMemset(p16, 0, cap * 2);
  cudaMemset(m, 0, n * 4);
  cudaMemset(v, 0, n * 4);
  CHECK(ratel_gen_theta0(theta, n, 0, ratel_gen_stream_key(0x5EED5EED, 1, 0, 0), NULL));

  ratel_config cfg;
  ratel_default_config(&cfg);
  CHECK(ratel_init(0, 0, 1, NULL, &cfg));
  ratel_range r;
  memset(&r, 0, sizeof r);
  r.param_bf16 = p16;
  r.grad_bf16 = g16;
  r.master = theta;
  r.exp_avg = m;
  r.exp_avg_sq = v;
  r.numel = n;
  r.apply_weight_decay = 1;
  CHECK(ratel_register_block(0, &r, 1, RATEL_DEVICE));

  cudaStream_t bwd;
  cudaStreamCreate(&bwd);
  for (int64_t t = 1; t <= 3; ++t) {
    CHECK(ratel_adam_step(1e-3, 0.9, 0.999, 1e-8, 1e-2, t));          /* arm first: AGO */
    CHECK(ratel_gen_grad16(g16, n, 0, ratel_gen_stream_key(0x5EED5EED, 2, t, 0), bwd)); /* "backward" */
    CHECK(ratel_offload_grad_chunk(0, bwd));                            /* the active message */
    CHECK(ratel_sync(bwd));                                             /* next forward ordered after */
  }
  cudaStreamSynchronize(bwd);

  float th[4];
  unsigned short pb[4];
  cudaMemcpy(th, theta + n - 4, sizeof th, cudaMemcpyDeviceToHost);
  cudaMemcpy(pb, (unsigned short*)p16 + n - 4, sizeof pb, cudaMemcpyDeviceToHost);
  int ok = 1;
  for (int i = 0; i < 4; ++i) {
    unsigned int u;
    memcpy(&u, &th[i], 4);
    unsigned short want = (unsigned short)((u + 0x7FFFu + ((u >> 16) & 1u)) >> 16);
    printf("theta[%llu] = %.8g  p16 = 0x%04x\n", (unsigned long long)(n - 4 + i), th[i], pb[i]);
    ok &= (pb[i] == want);
  }
  int64_t launches = ratel_launch_count();
  CHECK(ratel_finalize());
  printf("launches=%lld p16_matches_master=%d\n", (long long)launches, ok);
  return ok ? 0 : 2;
}
