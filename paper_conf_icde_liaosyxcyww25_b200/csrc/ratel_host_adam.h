// ratel_host_adam.h -- the paper-literal CPU handler (RATEL_HOST_COMPUTE).
//
// PAPER.md §IV-C: "the CPU updates the model states of the tensor i and
// produces a 16-bit parameter copy", on a CPU optimizer that
// keeps P32/OS32 in main memory.  This is that
// handler for one rank slice of one range: fp32 arithmetic (double for the
// Adam-L2 gradient) on the fp32 states in pinned host memory, bf16 RNE of the
// stored fp32 master.
#pragma once

#include <stddef.h>
#include <stdint.h>

namespace ratel {

struct HostAdamArgs {
  const uint16_t* g;   // bf16 grads (pinned host, copied D2H by the library)
  float* th;           // fp32 master   (pinned host, the caller's)
  float* m;            // fp32 exp_avg
  float* v;            // fp32 exp_avg_sq
  uint16_t* p;         // bf16 P16 out  (pinned host staging, copied H2D by the library)
  uint64_t n;
  int wd_on;
  int mode;            // RATEL_ADAMW / RATEL_ADAM_L2
  double lr, beta1, beta2, eps, wd, bc1, bc2, coef;
};

// Multi-threaded (OpenMP, `threads` <= 0: all available) elementwise update.
void host_adam_range(const HostAdamArgs& a, int threads);

}  // namespace ratel
