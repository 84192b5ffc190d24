// ratel_host_adam.cpp -- the CPU handler of RATEL_HOST_COMPUTE (see
// ratel_host_adam.h).  Runs inside a cudaLaunchHostFunc callback, so it must
// not call the CUDA API; it parallelises with OpenMP over 64K-element chunks.
#include "ratel_host_adam.h"

#include <omp.h>

#include <cmath>
#include <cstring>

#include "ratel.h"

namespace ratel {
namespace {

constexpr uint64_t kChunk = 1ull << 16;

inline uint16_t bf16_rne(float x) {
  uint32_t u;
  std::memcpy(&u, &x, sizeof u);
  if ((u & 0x7F800000u) == 0x7F800000u && (u & 0x007FFFFFu) != 0)
    return static_cast<uint16_t>((u >> 16) | 0x0040u);  // NaN stays a (quiet) NaN
  u += 0x7FFFu + ((u >> 16) & 1u);                       // round to nearest, ties to even
  return static_cast<uint16_t>(u >> 16);
}

// One chunk, double arithmetic on fp32 states.  Compiled for AVX-512, AVX2 and
// baseline x86-64; the loader picks the best the host CPU supports.
__attribute__((target_clones("avx512f", "avx2", "default")))
void chunk(const HostAdamArgs& a, uint64_t i0, uint64_t i1) {
  const double b1 = a.beta1, b2 = a.beta2, eps = a.eps;
  const double step = a.lr / a.bc1, inv_sqrt_bc2 = 1.0 / std::sqrt(a.bc2);
  const double decay = 1.0 - a.lr * a.wd;
  const bool adamw_wd = a.wd_on && a.mode == RATEL_ADAMW;
  const bool l2_wd = a.wd_on && a.mode == RATEL_ADAM_L2;
  for (uint64_t i = i0; i < i1; ++i) {
    const uint32_t gb = static_cast<uint32_t>(a.g[i]) << 16;
    float gf;
    std::memcpy(&gf, &gb, sizeof gf);
    double g = static_cast<double>(gf) * a.coef;
    double th = a.th[i];
    if (adamw_wd) th *= decay;
    if (l2_wd) g += a.wd * th;
    const double m = b1 * a.m[i] + (1.0 - b1) * g;
    const double v = b2 * a.v[i] + (1.0 - b2) * g * g;
    th -= step * m / (std::sqrt(v) * inv_sqrt_bc2 + eps);
    const float thf = static_cast<float>(th);
    a.th[i] = thf;
    a.m[i] = static_cast<float>(m);
    a.v[i] = static_cast<float>(v);
    a.p[i] = bf16_rne(thf);
  }
}

}  // namespace

void host_adam_range(const HostAdamArgs& a, int threads) {
  const uint64_t nchunks = (a.n + kChunk - 1) / kChunk;
  const int nt = threads > 0 ? threads : omp_get_max_threads();
#pragma omp parallel for schedule(static) num_threads(nt)
  for (int64_t c = 0; c < static_cast<int64_t>(nchunks); ++c) {
    const uint64_t i0 = static_cast<uint64_t>(c) * kChunk;
    const uint64_t i1 = i0 + kChunk < a.n ? i0 + kChunk : a.n;
    chunk(a, i0, i1);
  }
}

}  // namespace ratel
