// ratel_host_adam.cpp -- the CPU handler of RATEL_HOST_COMPUTE (see
// ratel_host_adam.h).  Runs inside a cudaLaunchHostFunc callback, so it must
// not call the CUDA API; it parallelises with OpenMP over 64K-element chunks,
// scheduled dynamically: with one team thread per core, the host's other
// threads (the caller, the CUDA driver) preempt some team thread, and a static
// split then waits for it (4.53 -> 5.03-5.08 G params/s on the 16-core box,
// profiles/r01_hostcompute_sweep.jsonl).
#include "ratel_host_adam.h"

#include <emmintrin.h>
#include <omp.h>

#include <cmath>
#include <cstring>

#include "ratel.h"

namespace ratel {
namespace {

constexpr uint64_t kChunk = 1ull << 16;

// P16 of a chunk is built in a thread-local buffer (128 KB, cache-resident)
// and written to the pinned staging with non-temporal 16-byte stores: the
// staging line is never read by the CPU, so a plain store's read-for-ownership
// (2 B/param of host DRAM traffic out of ~34) is avoided.
alignas(64) thread_local uint16_t t_p16[kChunk];

#ifndef RATEL_HOST_NT
#define RATEL_HOST_NT 1
#endif

void stream_out(uint16_t* dst, const uint16_t* src, uint64_t n) {
  uint64_t i = 0;
  if (!RATEL_HOST_NT) {   // A/B build: plain stores
    std::memcpy(dst, src, n * sizeof(uint16_t));
    return;
  }
  for (; i < n && (reinterpret_cast<uintptr_t>(dst + i) & 15u); ++i) dst[i] = src[i];
  for (; i + 8 <= n; i += 8)
    _mm_stream_si128(reinterpret_cast<__m128i*>(dst + i), _mm_loadu_si128(reinterpret_cast<const __m128i*>(src + i)));
  for (; i < n; ++i) dst[i] = src[i];
  _mm_sfence();   // globally visible before the callback returns and the H2D copy reads the staging
}

// fp32 arithmetic by default (the GPU kernel's precision; 4.0 vs 3.8 G params/s
// for double on the 16-core box, both within the R13 bounds); the L2 gradient
// is still formed in double (cancellation, R3).
#ifndef RATEL_HOST_FP32
#define RATEL_HOST_FP32 1
#endif

// One chunk on fp32 states (fp32 or double arithmetic), written so the compiler
// vectorises it (restrict pointers, branch-free bf16 rounding).  Compiled for
// AVX-512, AVX2 and baseline x86-64; the loader picks the best the CPU has.
__attribute__((target_clones("avx512f", "avx2", "default")))
void chunk(const HostAdamArgs& a, uint64_t i0, uint64_t i1) {
  const uint16_t* __restrict__ G = a.g;
  float* __restrict__ TH = a.th;
  float* __restrict__ M = a.m;
  float* __restrict__ V = a.v;
  uint16_t* __restrict__ P = t_p16;   // P[i - i0]: the thread-local chunk buffer
  const double b1 = a.beta1, b2 = a.beta2, omb1 = 1.0 - a.beta1, omb2 = 1.0 - a.beta2, eps = a.eps;
  const double step = a.lr / a.bc1, inv_sqrt_bc2 = 1.0 / std::sqrt(a.bc2), coef = a.coef;
  const double decay = (a.wd_on && a.mode == RATEL_ADAMW) ? 1.0 - a.lr * a.wd : 1.0;
  const double l2 = (a.wd_on && a.mode == RATEL_ADAM_L2) ? a.wd : 0.0;
#if RATEL_HOST_FP32
  // fp32 arithmetic (the GPU kernel's precision), twice the SIMD lanes of double
  const float b1f = static_cast<float>(b1), b2f = static_cast<float>(b2), omb1f = static_cast<float>(omb1),
              omb2f = static_cast<float>(omb2), epsf = static_cast<float>(eps), nstep = static_cast<float>(-step),
              isb = static_cast<float>(inv_sqrt_bc2), dec = static_cast<float>(decay);
  // No clip, no L2 term: fp32(double(g) * 1.0) == g exactly, so the widening
  // (half the SIMD lanes) is skipped -- same bits, a pure fp32 loop.
  const bool plain = coef == 1.0 && l2 == 0.0;
#pragma GCC ivdep
  for (uint64_t i = i0; i < i1; ++i) {
    uint32_t gb = static_cast<uint32_t>(G[i]) << 16;
    float gf;
    std::memcpy(&gf, &gb, sizeof gf);
    float th = TH[i];
    float g = gf;
    if (!plain) {   // loop-invariant: the compiler unswitches the loop
      double gd = static_cast<double>(gf) * coef;
      if (l2 != 0.0) gd += l2 * static_cast<double>(th);
      g = static_cast<float>(gd);
    }
    th *= dec;
    const float m = b1f * M[i] + omb1f * g;
    const float v = b2f * V[i] + omb2f * (g * g);
    th += nstep * (m / (std::sqrt(v) * isb + epsf));
    M[i] = m;
    V[i] = v;
    TH[i] = th;
    uint32_t u;
    std::memcpy(&u, &th, sizeof u);
    const uint32_t rne = (u + 0x7FFFu + ((u >> 16) & 1u)) >> 16;
    const bool nan = (u & 0x7FFFFFFFu) > 0x7F800000u;
    P[i - i0] = static_cast<uint16_t>(nan ? ((u >> 16) | 0x0040u) : rne);
  }
#else
#pragma GCC ivdep
  for (uint64_t i = i0; i < i1; ++i) {
    uint32_t gb = static_cast<uint32_t>(G[i]) << 16;
    float gf;
    std::memcpy(&gf, &gb, sizeof gf);
    double th = static_cast<double>(TH[i]);
    double g = static_cast<double>(gf) * coef;
    if (l2 != 0.0) g += l2 * th;   // Adam-L2 decay (loop-invariant test: the loop is unswitched)
    th *= decay;                   // AdamW decay (1 otherwise)
    const double m = b1 * M[i] + omb1 * g;
    const double v = b2 * V[i] + omb2 * g * g;
    th -= step * m / (std::sqrt(v) * inv_sqrt_bc2 + eps);
    const float thf = static_cast<float>(th);
    M[i] = static_cast<float>(m);
    V[i] = static_cast<float>(v);
    TH[i] = thf;
    uint32_t u;
    std::memcpy(&u, &thf, sizeof u);
    const uint32_t rne = (u + 0x7FFFu + ((u >> 16) & 1u)) >> 16;   // round to nearest, ties to even
    const bool nan = (u & 0x7FFFFFFFu) > 0x7F800000u;              // NaN stays a quiet NaN
    P[i - i0] = static_cast<uint16_t>(nan ? ((u >> 16) | 0x0040u) : rne);
  }
#endif
}

}  // namespace

void host_adam_range(const HostAdamArgs& a, int threads) {
  const uint64_t nchunks = (a.n + kChunk - 1) / kChunk;
  const int nt = threads > 0 ? threads : omp_get_max_threads();
#pragma omp parallel for schedule(dynamic, 1) num_threads(nt)
  for (int64_t c = 0; c < static_cast<int64_t>(nchunks); ++c) {
    const uint64_t i0 = static_cast<uint64_t>(c) * kChunk;
    const uint64_t i1 = i0 + kChunk < a.n ? i0 + kChunk : a.n;
    chunk(a, i0, i1);
    stream_out(a.p + i0, t_p16, i1 - i0);
  }
}

}  // namespace ratel
