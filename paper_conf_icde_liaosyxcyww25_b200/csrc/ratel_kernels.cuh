// ratel_kernels.cuh -- sm_100a kernels of the AGO optimizer step.
//
//   K1 adam_update_kernel   fused AdamW/Adam-L2 update + bf16 P16 emission
//                           (the handler of PAPER.md §IV-C: "the CPU updates
//                           the model states of the tensor i and produces a
//                           16-bit parameter copy")
//   K2 grad_sumsq_kernel    per-CTA partial sums of g^2 for the optional
//                           global-norm clip (reading R9)
//   K3 sumsq_finalize_kernel fixed-order reduction of the partials
//
// The path is elementwise and HBM-bound (28 B/param, ~0.6 flop/B): no tensor
// cores.  K1 streams five SoA arrays with 128-bit loads/stores through a
// grid-stride loop sized to the SMs, and every element -- vector body or
// scalar tail -- goes through the SAME adam_update() with explicit
// __fmaf_rn/__fmul_rn (and sqrt.approx/rcp.approx, or __fsqrt_rn/__fdiv_rn with
// RATEL_K1_FASTMATH=0; R7), so the compiler cannot contract
// differently in the two paths.  That makes results bitwise identical across
// world size, tile size, residency and hand-off order (R16).
#pragma once

#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "ratel.h"
#include "ratel_bf16.cuh"

namespace ratel {

constexpr int kMaxRanges = RATEL_MAX_RANGES_PER_BLOCK;
constexpr int kThreads = 256;

// Per-step scalars, derived on the host in double and rounded once to fp32.
struct AdamScalars {
  float beta1, one_minus_beta1;   // b1, 1-b1
  float beta2, one_minus_beta2;   // b2, 1-b2
  float neg_step_size;            // -lr / (1 - b1^t)
  float inv_sqrt_bc2;             // 1 / sqrt(1 - b2^t)
  float eps;
  float decay;                    // 1 - lr*wd      (AdamW)
  float wd;                       // wd             (unused; kept for layout clarity)
  double wd_d;                    // wd in double   (Adam-L2, see adam_update)
};

// One rank-slice (or one staged tile) of a parameter range.
struct RangeDesc {
  const uint16_t* g;  // bf16 grads of the slice
  float* th;          // fp32 master
  float* m;           // fp32 exp_avg
  float* v;           // fp32 exp_avg_sq
  uint16_t* p;        // bf16 working copy of the slice
  uint64_t n;         // elements
  int wd_on;
  int pad_;
};

// Fused all-gather over peer memory: this rank's P16 slice is also stored
// straight into every other rank's P16 buffer (NVLink P2P stores) --
// pointers already offset to the slice start of this range.
constexpr int kMaxPeers = 8;
struct PeerDesc {
  uint16_t* p[kMaxPeers];
  int n;
};

struct UpdateParams {
  RangeDesc r[kMaxRanges];
  PeerDesc peers[kMaxRanges];
  int nr;
  int any_peers;
  AdamScalars s;
  const double* sumsq;   // clip: global sum of g^2 (device); unused otherwise
  double max_norm;
  int* nonfinite_flag;   // clip: set to !isfinite(sumsq) by CTA 0
  // TMA kernel tile scheduler: NULL = static round robin; else tiles are
  // taken dynamically, tile = atomicAdd(tile_ctr, 1) - tile_base (the
  // counter only grows; one launch advances it by tiles + grid).
  unsigned long long* tile_ctr;
  unsigned long long tile_base;
  // > 0: non-persistent grid, CTA b takes tiles [b*cta_tiles, (b+1)*cta_tiles)
  // (tile_ctr is then NULL); 0: persistent grid.
  uint32_t cta_tiles;
};

struct SumsqParams {
  const uint16_t* g[kMaxRanges];
  uint64_t n[kMaxRanges];
  int nr;
  double* partials;  // one slot per CTA
};

#ifndef RATEL_K1_NOMATH
#define RATEL_K1_NOMATH 0
#endif
#ifndef RATEL_K1_FASTMATH
#define RATEL_K1_FASTMATH 1
#endif

// The per-element update.  Explicit-rounding intrinsics fix the operation
// sequence (no contraction freedom):
//   AdamW:   theta = theta*decay            (wd_on)
//   Adam-L2: g     = fp32(g*coef + wd*theta, formed in fp64)   (wd_on)
// The L2 term is formed in double: g and wd*theta cancel when the gradient
// balances the decay, and fp32(wd) alone (rel. error 2e-8) would then move
// g' by more than its own ulp and the update by >1e-5 of its scale near
// |g'| ~ eps (measured on B200; R3); with clipping the fp32
// rounding of g*coef did the same to v (measured).  Two fp64 ops per element
// are far inside the ALU budget of this HBM-bound kernel.
//   m     = fma(b1, m, (1-b1)*g)
//   v     = fma(b2, v, (1-b2)*(g*g))        g*g is exact for a bf16 g
//   denom = fma(sqrt(v), 1/sqrt(bc2), eps)  == sqrt(v/bc2) + eps
//   theta = fma(-lr/bc1, m/denom, theta)
template <int MODE, bool CLIP>
__device__ __forceinline__ void adam_update(float g, float& th, float& m, float& v, const AdamScalars& s,
                                            bool wd_on, float coef_f, double coef_d) {
  if (MODE == RATEL_ADAM_L2) {
    // g' = g*coef + wd*theta in double, rounded once: the two terms cancel
    // when the gradient balances the decay (see the comment above).
    double gd = static_cast<double>(g);
    if (CLIP) gd *= coef_d;
    if (wd_on) gd = __fma_rn(s.wd_d, static_cast<double>(th), gd);
    g = __double2float_rn(gd);
  } else {
    if (CLIP) g = __fmul_rn(g, coef_f);
    if (wd_on) th = __fmul_rn(th, s.decay);
  }
  m = __fmaf_rn(s.beta1, m, __fmul_rn(s.one_minus_beta1, g));
  v = __fmaf_rn(s.beta2, v, __fmul_rn(s.one_minus_beta2, __fmul_rn(g, g)));
#if RATEL_K1_FASTMATH
  float sq, r;
  asm("sqrt.approx.f32 %0, %1;" : "=f"(sq) : "f"(v));
  const float denom = __fmaf_rn(sq, s.inv_sqrt_bc2, s.eps);
  asm("rcp.approx.f32 %0, %1;" : "=f"(r) : "f"(denom));
  th = __fmaf_rn(s.neg_step_size, __fmul_rn(m, r), th);
#else
  const float denom = __fmaf_rn(__fsqrt_rn(v), s.inv_sqrt_bc2, s.eps);
  th = __fmaf_rn(s.neg_step_size, __fdiv_rn(m, denom), th);
#endif
}

// ---- K1 memory operations --------------------------------------------------
// Build-time variants (tools/k1_sweep.py measures them on the B200):
//   RATEL_K1_LDST 0: 2 x 128-bit ld/st.global.cs per fp32 octet
//                 1: 256-bit ld/st (sm_100) with L1::no_allocate + L2::evict_first
//                 2: 256-bit ld/st, no cache hints
//   RATEL_K1_UNROLL  octets in flight per thread per loop trip
//   RATEL_K1_MINB    __launch_bounds__ min CTAs/SM (register budget)
#ifndef RATEL_K1_LDST
#define RATEL_K1_LDST 2
#endif
#ifndef RATEL_K1_UNROLL
#define RATEL_K1_UNROLL 2
#endif
#ifndef RATEL_K1_MINB
#define RATEL_K1_MINB 2
#endif

__device__ __forceinline__ void ld_f8(const float* p, float (&r)[8]) {
#if RATEL_K1_LDST == 0
  const float4 a = __ldcs(reinterpret_cast<const float4*>(p));
  const float4 b = __ldcs(reinterpret_cast<const float4*>(p) + 1);
  r[0] = a.x; r[1] = a.y; r[2] = a.z; r[3] = a.w; r[4] = b.x; r[5] = b.y; r[6] = b.z; r[7] = b.w;
#elif RATEL_K1_LDST == 1
  asm volatile("ld.global.L1::no_allocate.L2::evict_first.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(r[0]), "=f"(r[1]), "=f"(r[2]), "=f"(r[3]), "=f"(r[4]), "=f"(r[5]), "=f"(r[6]), "=f"(r[7])
               : "l"(p));
#else
  asm volatile("ld.global.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(r[0]), "=f"(r[1]), "=f"(r[2]), "=f"(r[3]), "=f"(r[4]), "=f"(r[5]), "=f"(r[6]), "=f"(r[7])
               : "l"(p));
#endif
}

__device__ __forceinline__ void st_f8(float* p, const float (&r)[8]) {
#if RATEL_K1_LDST == 0
  __stcs(reinterpret_cast<float4*>(p), make_float4(r[0], r[1], r[2], r[3]));
  __stcs(reinterpret_cast<float4*>(p) + 1, make_float4(r[4], r[5], r[6], r[7]));
#elif RATEL_K1_LDST == 1
  asm volatile("st.global.L1::no_allocate.L2::evict_first.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};"
               :: "l"(p), "f"(r[0]), "f"(r[1]), "f"(r[2]), "f"(r[3]), "f"(r[4]), "f"(r[5]), "f"(r[6]), "f"(r[7])
               : "memory");
#else
  asm volatile("st.global.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};"
               :: "l"(p), "f"(r[0]), "f"(r[1]), "f"(r[2]), "f"(r[3]), "f"(r[4]), "f"(r[5]), "f"(r[6]), "f"(r[7])
               : "memory");
#endif
}

__device__ __forceinline__ uint4 ld_g8(const uint16_t* p) {
#if RATEL_K1_LDST != 2  // (.L2::evict_first exists only for 256-bit accesses)
  return __ldcs(reinterpret_cast<const uint4*>(p));
#else
  return *reinterpret_cast<const uint4*>(p);
#endif
}

__device__ __forceinline__ void st_peers8(const PeerDesc& pd, uint64_t elem, uint4 v) {
  for (int q = 0; q < pd.n; ++q)
    asm volatile("st.global.v4.b32 [%0], {%1,%2,%3,%4};" ::"l"(pd.p[q] + elem), "r"(v.x), "r"(v.y),
                 "r"(v.z), "r"(v.w) : "memory");
}

__device__ __forceinline__ void st_p8(uint16_t* p, uint4 v) {
#if RATEL_K1_LDST == 2
  *reinterpret_cast<uint4*>(p) = v;
#else
  __stcs(reinterpret_cast<uint4*>(p), v);
#endif
}

// 8 consecutive elements: 16 B of g, 32 B each of theta, m, v.
struct Frag8 {
  uint4 g;
  float t[8], m[8], v[8];
};

__device__ __forceinline__ void load8(Frag8& f, const RangeDesc& R, uint64_t i) {
  f.g = ld_g8(R.g + 8 * i);
  ld_f8(R.th + 8 * i, f.t);
  ld_f8(R.m + 8 * i, f.m);
  ld_f8(R.v + 8 * i, f.v);
}

// Update octet i of R from the fp32 gradients g[0..7] (f.g unused) and
// store theta, m, v, P16 (and the peer P16 copies).
template <int MODE, bool CLIP>
__device__ __forceinline__ void update_store8_g(const float (&g)[8], Frag8& f, const RangeDesc& R, uint64_t i,
                                                const AdamScalars& s, float coef_f, double coef_d,
                                                const PeerDesc& pd) {
  const bool wd = R.wd_on != 0;
#pragma unroll
  for (int k = 0; k < 8; ++k) adam_update<MODE, CLIP>(g[k], f.t[k], f.m[k], f.v[k], s, wd, coef_f, coef_d);
  st_f8(R.th + 8 * i, f.t);
  st_f8(R.m + 8 * i, f.m);
  st_f8(R.v + 8 * i, f.v);
  uint4 pk;
  pk.x = pack_bf16x2_rn(f.t[0], f.t[1]);
  pk.y = pack_bf16x2_rn(f.t[2], f.t[3]);
  pk.z = pack_bf16x2_rn(f.t[4], f.t[5]);
  pk.w = pack_bf16x2_rn(f.t[6], f.t[7]);
  st_p8(R.p + 8 * i, pk);
  st_peers8(pd, 8 * i, pk);
}

template <int MODE, bool CLIP>
__device__ __forceinline__ void update_store8(Frag8& f, const RangeDesc& R, uint64_t i,
                                              const AdamScalars& s, float coef_f, double coef_d,
                                              const PeerDesc& pd) {
  const uint32_t gw[4] = {f.g.x, f.g.y, f.g.z, f.g.w};
  float g[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    const uint32_t w = gw[k >> 1];
    g[k] = bf16_bits_to_f32((k & 1) ? (w >> 16) : (w & 0xFFFFu));
  }
  update_store8_g<MODE, CLIP>(g, f, R, i, s, coef_f, coef_d, pd);
}

template <int MODE, bool CLIP>
__device__ __forceinline__ void update_scalar(const RangeDesc& R, uint64_t j, const AdamScalars& s,
                                              float coef_f, double coef_d, const PeerDesc& pd) {
  float g = bf16_bits_to_f32(R.g[j]);
  float th = R.th[j], m = R.m[j], v = R.v[j];
  adam_update<MODE, CLIP>(g, th, m, v, s, R.wd_on != 0, coef_f, coef_d);
  R.th[j] = th;
  R.m[j] = m;
  R.v[j] = v;
  const uint16_t pb = static_cast<uint16_t>(pack_bf16x2_rn(th, 0.0f) & 0xFFFFu);
  R.p[j] = pb;
  for (int q = 0; q < pd.n; ++q) pd.p[q][j] = pb;
}

__device__ __forceinline__ double clip_coef_from(const double* sumsq, double max_norm, int* flag) {
  const double S = *sumsq;
  double c = max_norm / (sqrt(S) + 1e-6);
  c = (c < 1.0 || isnan(c)) ? c : 1.0;  // torch: clamp(max=1), NaN propagates
  if (flag != nullptr && blockIdx.x == 0 && threadIdx.x == 0) *flag = isfinite(S) ? 0 : 1;
  return c;
}

// K1.  Grid-stride over 8-element octets of each range, RATEL_K1_UNROLL
// octets in flight per thread (all their loads issued before any math), then
// the < 8-element scalar tail.
// U / MINB: the default build (2 octets in flight, 2 CTAs/SM) or the "lite"
// variant (cfg.k1_kernel = RATEL_UPDATE_LDG_LITE: 1 octet, 4 CTAs/SM, <= 64
// registers, no shared memory) whose CTAs fit beside a backward GEMM CTA on
// the same SM.
template <int MODE, bool CLIP, int U = RATEL_K1_UNROLL, int MINB = RATEL_K1_MINB>
__global__ void __launch_bounds__(kThreads, MINB) adam_update_kernel(const __grid_constant__ UpdateParams P) {
  const double coef_d = CLIP ? clip_coef_from(P.sumsq, P.max_norm, P.nonfinite_flag) : 1.0;
  const float coef_f = static_cast<float>(coef_d);
  const uint64_t tid = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
  for (int r = 0; r < P.nr; ++r) {
    const RangeDesc R = P.r[r];
    const uint64_t n8 = R.n >> 3;
    uint64_t i = tid;
    for (; i + (U - 1) * stride < n8; i += U * stride) {
      Frag8 f[U];
#pragma unroll
      for (int u = 0; u < U; ++u) load8(f[u], R, i + u * stride);
#pragma unroll
      for (int u = 0; u < U; ++u) update_store8<MODE, CLIP>(f[u], R, i + u * stride, P.s, coef_f, coef_d, P.peers[r]);
    }
    for (; i < n8; i += stride) {
      Frag8 f;
      load8(f, R, i);
      update_store8<MODE, CLIP>(f, R, i, P.s, coef_f, coef_d, P.peers[r]);
    }
    const uint64_t j = (n8 << 3) + tid;
    if (j < R.n) update_scalar<MODE, CLIP>(R, j, P.s, coef_f, coef_d, P.peers[r]);
  }
  if (P.any_peers) __threadfence_system();  // peer P16 stores visible before the step's barrier
}

// ---- K1, TMA-staged variant ------------------------------------------------
// One CTA per SM (persistent).  A producer warp streams each tile's g, theta,
// m, v into a ring of shared-memory stages with 1-D bulk copies
// (cp.async.bulk, completion on an mbarrier); consumer warps run the same
// adam_update() per element from shared memory and write theta, m, v, P16
// straight to global with 256-bit stores.  Bytes in flight are bounded by the
// stage ring (RATEL_TMA_STAGES x 14 B x tile), not by registers.
#ifndef RATEL_TMA_CONSUMER_WARPS
#define RATEL_TMA_CONSUMER_WARPS 16
#endif
#ifndef RATEL_TMA_STAGES
#define RATEL_TMA_STAGES 4
#endif
// How a stage goes back to the producer (measured: profiles/sweeps/,
// profiles/r01_racecheck_*.log):
//   0 lane 0 arrives right after __syncwarp -- RACY: the TMA refill overwrote
//     smem that other lanes' loads had not returned yet (capped-grid tests);
//   1 every consumer thread arrives (racecheck-clean);
//   2 lane 0 arrives after the warp CONSUMED the values (correct by data
//     dependence, but racecheck cannot see that and flags it);
//   3 fence.proxy.async + lane 0 (flagged by racecheck as well);
//   4 default: results are written back into the stage and bulk-stored by one
//     thread (cp.async.bulk global<-shared); that thread releases a stage once
//     cp.async.bulk.wait_group.read says the store finished reading it.
//     Racecheck-clean and the fastest (fewer STG instructions).
#ifndef RATEL_TMA_EVICT_FIRST
#define RATEL_TMA_EVICT_FIRST 0
#endif
#ifndef RATEL_TMA_CTAS_PER_SM
#define RATEL_TMA_CTAS_PER_SM 1
#endif
#ifndef RATEL_TMA_RELEASE
#define RATEL_TMA_RELEASE 4
#endif
constexpr int kTmaConsumerWarps = RATEL_TMA_CONSUMER_WARPS;
constexpr int kTmaThreads = 32 * (kTmaConsumerWarps + 1);
constexpr int kTmaTile = kTmaConsumerWarps * 32 * 8;          // elements per tile (1 octet per consumer thread)
constexpr int kTmaStages = RATEL_TMA_STAGES;
constexpr uint32_t kTmaStageBytes = kTmaTile * 14;            // g 2 + theta/m/v 12
constexpr uint32_t kTmaSmemBytes = kTmaStages * kTmaStageBytes + 3 * kTmaStages * 8;  // + full/empty/tile id

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}\n" ::"r"(smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ void bulk_load(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
#if RATEL_TMA_EVICT_FIRST
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
               ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol) : "memory");
#else
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
#endif
}

__device__ __forceinline__ void bulk_store(void* dst, const void* src, uint32_t bytes) {
#if RATEL_TMA_EVICT_FIRST
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;"
               ::"l"(dst), "r"(smem_u32(src)), "r"(bytes), "l"(pol) : "memory");
#else
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
               ::"l"(dst), "r"(smem_u32(src)), "r"(bytes) : "memory");
#endif
}

// Tile k of the concatenation of the ranges' vector bodies (n & ~7 each).
struct TileLoc {
  int r;
  uint64_t off;
  uint32_t len;
};
__device__ __forceinline__ TileLoc locate_tile(const UpdateParams& P, uint64_t k) {
  TileLoc t{0, 0, 0};
  for (int r = 0; r < P.nr; ++r) {
    const uint64_t body = P.r[r].n & ~7ull;
    const uint64_t nt = (body + kTmaTile - 1) / kTmaTile;
    if (k < nt) {
      t.r = r;
      t.off = k * kTmaTile;
      t.len = static_cast<uint32_t>(body - t.off < (uint64_t)kTmaTile ? body - t.off : kTmaTile);
      return t;
    }
    k -= nt;
  }
  t.r = -1;
  return t;
}

template <int MODE, bool CLIP>
__global__ void __launch_bounds__(kTmaThreads, RATEL_TMA_CTAS_PER_SM) adam_update_tma_kernel(const __grid_constant__ UpdateParams P) {
  extern __shared__ __align__(128) uint8_t smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + kTmaStages * kTmaStageBytes);
  uint64_t* empty = full + kTmaStages;
  volatile uint64_t* tile_id = empty + kTmaStages;  // the producer's tile per stage (~0 = no more)
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < kTmaStages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], RATEL_TMA_RELEASE == 1 ? 32 * kTmaConsumerWarps
                           : (RATEL_TMA_RELEASE == 4 ? 1 : kTmaConsumerWarps));
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  __syncthreads();
  uint64_t total = 0;
  for (int r = 0; r < P.nr; ++r) total += ((P.r[r].n & ~7ull) + kTmaTile - 1) / kTmaTile;

  if (warp == kTmaConsumerWarps) {  // producer
    if (lane == 0) {
      // Dynamic scheduling: CTAs that run ahead take more tiles, so all SMs
      // finish together (a static split left the slowest SM's tail exposed;
      // measured in DESIGN.md §6).  The next grab is issued one tile early so
      // its latency overlaps the wait for a free stage.
      const bool dyn = P.tile_ctr != nullptr;
      const uint64_t Y = P.cta_tiles;
      uint64_t k = Y ? blockIdx.x * Y : dyn ? atomicAdd(P.tile_ctr, 1ull) - P.tile_base : blockIdx.x;
      const uint64_t lim = Y ? (k + Y < total ? k + Y : total) : total;
      int stage = 0;
      uint32_t phase = 0;
      for (;;) {
        uint64_t kn = k;
        if (k < lim) kn = Y ? k + 1 : dyn ? atomicAdd(P.tile_ctr, 1ull) - P.tile_base : k + gridDim.x;
        mbar_wait(&empty[stage], phase ^ 1);
        if (k >= lim) {  // no more tiles: tell the consumers
          tile_id[stage] = ~0ull;
          mbar_arrive(&full[stage]);
          break;
        }
        tile_id[stage] = k;
        const TileLoc t = locate_tile(P, k);
        const RangeDesc& R = P.r[t.r];
        uint8_t* base = smem + stage * kTmaStageBytes;
        mbar_expect_tx(&full[stage], t.len * 14u);
        bulk_load(base, R.g + t.off, t.len * 2u, &full[stage]);
        bulk_load(base + kTmaTile * 2, R.th + t.off, t.len * 4u, &full[stage]);
        bulk_load(base + kTmaTile * 6, R.m + t.off, t.len * 4u, &full[stage]);
        bulk_load(base + kTmaTile * 10, R.v + t.off, t.len * 4u, &full[stage]);
        if (++stage == kTmaStages) {
          stage = 0;
          phase ^= 1;
        }
        k = kn;
      }
    }
  } else {  // consumers
    const double coef_d = CLIP ? clip_coef_from(P.sumsq, P.max_norm, P.nonfinite_flag) : 1.0;
    const float coef_f = static_cast<float>(coef_d);
    int stage = 0;
    uint32_t phase = 0;
    int prev_stage = -1;
    (void)prev_stage;
    const uint32_t o = threadIdx.x;  // octet within the tile
    for (;;) {
      mbar_wait(&full[stage], phase);
      const uint64_t k = tile_id[stage];
      if (k == ~0ull) break;
      const TileLoc t = locate_tile(P, k);
      const RangeDesc& R = P.r[t.r];
      const uint8_t* base = smem + stage * kTmaStageBytes;
      const bool valid = 8 * o < t.len;
      Frag8 f;
      if (valid) {
        f.g = *reinterpret_cast<const uint4*>(base + 16 * o);
        const float4* th = reinterpret_cast<const float4*>(base + kTmaTile * 2) + 2 * o;
        const float4* mm = reinterpret_cast<const float4*>(base + kTmaTile * 6) + 2 * o;
        const float4* vv = reinterpret_cast<const float4*>(base + kTmaTile * 10) + 2 * o;
        const float4 t0 = th[0], t1 = th[1], m0 = mm[0], m1 = mm[1], v0 = vv[0], v1 = vv[1];
        f.t[0] = t0.x; f.t[1] = t0.y; f.t[2] = t0.z; f.t[3] = t0.w;
        f.t[4] = t1.x; f.t[5] = t1.y; f.t[6] = t1.z; f.t[7] = t1.w;
        f.m[0] = m0.x; f.m[1] = m0.y; f.m[2] = m0.z; f.m[3] = m0.w;
        f.m[4] = m1.x; f.m[5] = m1.y; f.m[6] = m1.z; f.m[7] = m1.w;
        f.v[0] = v0.x; f.v[1] = v0.y; f.v[2] = v0.z; f.v[3] = v0.w;
        f.v[4] = v1.x; f.v[5] = v1.y; f.v[6] = v1.z; f.v[7] = v1.w;
      }
#if RATEL_TMA_RELEASE == 0
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[stage]);  // the stage's data is in registers now
      if (valid) update_store8<MODE, CLIP>(f, R, (t.off >> 3) + o, P.s, coef_f, coef_d, P.peers[t.r]);
#elif RATEL_TMA_RELEASE == 1
      mbar_arrive(&empty[stage]);                 // every consumer thread arrives
      if (valid) update_store8<MODE, CLIP>(f, R, (t.off >> 3) + o, P.s, coef_f, coef_d, P.peers[t.r]);
#elif RATEL_TMA_RELEASE == 2
      if (valid) update_store8<MODE, CLIP>(f, R, (t.off >> 3) + o, P.s, coef_f, coef_d, P.peers[t.r]);
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[stage]);  // after the values were consumed
#elif RATEL_TMA_RELEASE == 3
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[stage]);
      if (valid) update_store8<MODE, CLIP>(f, R, (t.off >> 3) + o, P.s, coef_f, coef_d, P.peers[t.r]);
#else  // 4: results written back into the stage, bulk-stored by one thread
      if (valid) {
        const bool wd = R.wd_on != 0;
        const uint32_t gw[4] = {f.g.x, f.g.y, f.g.z, f.g.w};
#pragma unroll
        for (int kk = 0; kk < 8; ++kk) {
          const uint32_t w = gw[kk >> 1];
          float g = bf16_bits_to_f32((kk & 1) ? (w >> 16) : (w & 0xFFFFu));
#if RATEL_K1_NOMATH  // diagnostic build only: pure data movement through the same pipeline
          f.t[kk] += g * 0.0f;
#else
          adam_update<MODE, CLIP>(g, f.t[kk], f.m[kk], f.v[kk], P.s, wd, coef_f, coef_d);
#endif
        }
        uint8_t* wb = smem + stage * kTmaStageBytes;
        float4* th = reinterpret_cast<float4*>(wb + kTmaTile * 2) + 2 * o;
        float4* mm = reinterpret_cast<float4*>(wb + kTmaTile * 6) + 2 * o;
        float4* vv = reinterpret_cast<float4*>(wb + kTmaTile * 10) + 2 * o;
        th[0] = make_float4(f.t[0], f.t[1], f.t[2], f.t[3]);
        th[1] = make_float4(f.t[4], f.t[5], f.t[6], f.t[7]);
        mm[0] = make_float4(f.m[0], f.m[1], f.m[2], f.m[3]);
        mm[1] = make_float4(f.m[4], f.m[5], f.m[6], f.m[7]);
        vv[0] = make_float4(f.v[0], f.v[1], f.v[2], f.v[3]);
        vv[1] = make_float4(f.v[4], f.v[5], f.v[6], f.v[7]);
        uint4 pk;
        pk.x = pack_bf16x2_rn(f.t[0], f.t[1]);
        pk.y = pack_bf16x2_rn(f.t[2], f.t[3]);
        pk.z = pack_bf16x2_rn(f.t[4], f.t[5]);
        pk.w = pack_bf16x2_rn(f.t[6], f.t[7]);
        *reinterpret_cast<uint4*>(wb + 16 * o) = pk;
        st_peers8(P.peers[t.r], t.off + 8 * o, pk);  // fused all-gather: NVLink P2P stores
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic smem writes -> async proxy
      asm volatile("bar.sync 1, %0;" ::"r"(kTmaConsumerWarps * 32) : "memory");
      if (threadIdx.x == 0) {
        uint8_t* wb = smem + stage * kTmaStageBytes;
        bulk_store(R.th + t.off, wb + kTmaTile * 2, t.len * 4u);
        bulk_store(R.m + t.off, wb + kTmaTile * 6, t.len * 4u);
        bulk_store(R.v + t.off, wb + kTmaTile * 10, t.len * 4u);
        bulk_store(R.p + t.off, wb, t.len * 2u);
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");  // previous tile's stores read smem
        if (prev_stage >= 0) mbar_arrive(&empty[prev_stage]);
        prev_stage = stage;
      }
#endif
      if (++stage == kTmaStages) {
        stage = 0;
        phase ^= 1;
      }
    }
#if RATEL_TMA_RELEASE == 4
    if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
#endif
    // scalar tails (< 8 elements per range), CTA 0
    if (blockIdx.x == 0) {
      for (int r = 0; r < P.nr; ++r) {
        const uint64_t j = (P.r[r].n & ~7ull) + threadIdx.x;
        if (j < P.r[r].n) update_scalar<MODE, CLIP>(P.r[r], j, P.s, coef_f, coef_d, P.peers[r]);
      }
    }
    if (P.any_peers) __threadfence_system();  // peer P16 stores visible before the step's barrier
  }
}

// ---- K1-RS: the data-parallel gradient reduction fused into the update ------
// (R17).  Each rank keeps its local full-range G16;
// for its own slice the kernel loads the N ranks' bf16 octets (the peers'
// over NVLink, P2P), sums them in fp64 in rank order, scales once and rounds
// once to fp32, then runs the same adam_update().  This replaces the
// reduce-scatter: no reduced-gradient buffer, no separate NCCL kernel.  A
// range without peer grads is the n = 1, scale = 1 case, which reproduces
// the plain path bit for bit (fp32(1.0 * bf16) == bf16).  Register-staged
// (LDG) like adam_update_kernel: on a real multi-GPU system the kernel is
// bound by the 2(N-1)/N B/param of NVLink reads, not by HBM.
constexpr int kMaxRanks = 8;
struct GradPeers {
  const uint16_t* g[kMaxRanks];  // every rank's G16, offset to this slice/tile, rank order
  int n;                          // ranks summed (>= 1)
  int pad_;
  double scale;                   // 1/N = data-parallel mean, 1 = sum
};
struct RsUpdateParams {
  UpdateParams u;
  GradPeers gp[kMaxRanges];
};
struct RsSumsqParams {
  GradPeers gp[kMaxRanges];
  uint64_t n[kMaxRanges];
  int nr;
  double* partials;  // one slot per CTA
};

__device__ __forceinline__ void reduce_g8(const GradPeers& gp, uint64_t e, float (&g)[8]) {
  uint4 w[kMaxRanks];
#pragma unroll
  for (int q = 0; q < kMaxRanks; ++q)
    if (q < gp.n) w[q] = *reinterpret_cast<const uint4*>(gp.g[q] + e);
  double s[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) s[k] = 0.0;
#pragma unroll
  for (int q = 0; q < kMaxRanks; ++q) {
    if (q < gp.n) {
      const uint32_t ws[4] = {w[q].x, w[q].y, w[q].z, w[q].w};
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        s[2 * k] = __dadd_rn(s[2 * k], static_cast<double>(bf16_bits_to_f32(ws[k] & 0xFFFFu)));
        s[2 * k + 1] = __dadd_rn(s[2 * k + 1], static_cast<double>(bf16_bits_to_f32(ws[k] >> 16)));
      }
    }
  }
#pragma unroll
  for (int k = 0; k < 8; ++k) g[k] = __double2float_rn(__dmul_rn(s[k], gp.scale));
}

__device__ __forceinline__ float reduce_g1(const GradPeers& gp, uint64_t j) {
  double s = 0.0;
  for (int q = 0; q < gp.n; ++q) s = __dadd_rn(s, static_cast<double>(bf16_bits_to_f32(gp.g[q][j])));
  return __double2float_rn(__dmul_rn(s, gp.scale));
}

// Tiles of kRsTile elements of the ranges' vector bodies, taken dynamically
// from the same per-stream counter as the TMA kernel (tile = atomicAdd - base,
// the next grab issued while the current tile is processed); each thread
// updates kRsTile / 8 / kThreads octets of a tile.
constexpr int kRsTile = 4096;
static_assert(kRsTile % (8 * kThreads) == 0, "RS tile = whole octets per thread");

__device__ __forceinline__ TileLoc locate_rs_tile(const UpdateParams& P, uint64_t k) {
  TileLoc t{0, 0, 0};
  for (int r = 0; r < P.nr; ++r) {
    const uint64_t body = P.r[r].n & ~7ull;
    const uint64_t nt = (body + kRsTile - 1) / kRsTile;
    if (k < nt) {
      t.r = r;
      t.off = k * kRsTile;
      t.len = static_cast<uint32_t>(body - t.off < (uint64_t)kRsTile ? body - t.off : kRsTile);
      return t;
    }
    k -= nt;
  }
  t.r = -1;
  return t;
}

template <int MODE, bool CLIP>
__global__ void __launch_bounds__(kThreads, RATEL_K1_MINB) adam_update_rs_kernel(const __grid_constant__ RsUpdateParams Q) {
  const UpdateParams& P = Q.u;
  const double coef_d = CLIP ? clip_coef_from(P.sumsq, P.max_norm, P.nonfinite_flag) : 1.0;
  const float coef_f = static_cast<float>(coef_d);
  uint64_t total = 0;
  for (int r = 0; r < P.nr; ++r) total += ((P.r[r].n & ~7ull) + kRsTile - 1) / kRsTile;
  __shared__ uint64_t s_next;
  const bool dyn = P.tile_ctr != nullptr;
  if (threadIdx.x == 0) s_next = dyn ? atomicAdd(P.tile_ctr, 1ull) - P.tile_base : blockIdx.x;
  for (;;) {
    __syncthreads();
    const uint64_t k = s_next;
    __syncthreads();
    if (k >= total) break;
    if (threadIdx.x == 0) s_next = dyn ? atomicAdd(P.tile_ctr, 1ull) - P.tile_base : k + gridDim.x;
    const TileLoc t = locate_rs_tile(P, k);
    const RangeDesc& R = P.r[t.r];
    const GradPeers& gp = Q.gp[t.r];
#pragma unroll
    for (int u = 0; u < kRsTile / (8 * kThreads); ++u) {
      const uint32_t o = threadIdx.x + u * kThreads;  // octet within the tile
      if (8 * o < t.len) {
        const uint64_t i = (t.off >> 3) + o;
        Frag8 f;
        ld_f8(R.th + 8 * i, f.t);
        ld_f8(R.m + 8 * i, f.m);
        ld_f8(R.v + 8 * i, f.v);
        float g[8];
        reduce_g8(gp, 8 * i, g);
        update_store8_g<MODE, CLIP>(g, f, R, i, P.s, coef_f, coef_d, P.peers[t.r]);
      }
    }
  }
  // scalar tails (< 8 elements per range), CTA 0
  for (int r = 0; r < P.nr && blockIdx.x == 0; ++r) {
    const RangeDesc& R = P.r[r];
    const GradPeers& gp = Q.gp[r];
    const uint64_t j = (R.n & ~7ull) + threadIdx.x;
    if (j < R.n) {
      float th = R.th[j], m = R.m[j], v = R.v[j];
      adam_update<MODE, CLIP>(reduce_g1(gp, j), th, m, v, P.s, R.wd_on != 0, coef_f, coef_d);
      R.th[j] = th;
      R.m[j] = m;
      R.v[j] = v;
      const uint16_t pb = static_cast<uint16_t>(pack_bf16x2_rn(th, 0.0f) & 0xFFFFu);
      R.p[j] = pb;
      const PeerDesc& pd = P.peers[r];
      for (int q = 0; q < pd.n; ++q) pd.p[q][j] = pb;
    }
  }
  if (P.any_peers) __threadfence_system();
}

// ---- K1-RS, TMA-staged variant (default with cfg.k1_kernel = TMA) ----------
// The fused reduction with K1's data movement: a producer warp bulk-copies,
// per 2048-element tile, every rank's G16 (the peers' through their P2P
// mappings -- TMA keeps a stage's worth of NVLink reads in flight per SM
// instead of a few registers' worth) plus theta, m, v into a shared-memory
// ring of ~224 KB (8 stages at N = 1 down to 4 at N = 8); 8 consumer warps reduce the N gradients of their octet
// in fp64 in rank order (reduce_g8's arithmetic, so the result is bitwise the
// LDG kernel's), update, write theta/m/v and P16 back into the stage, and one
// thread bulk-stores them (K1's release protocol 4).  Stage layout for nmax
// = the largest rank count among the launch's ranges:
//   [G16 rank 0 .. rank nmax-1 : 2 B x tile each][theta][m][v : 4 B x tile]
// P16 is written over rank 0's G16 octet by the thread that read it.
constexpr int kRsTmaConsumerWarps = 8;
constexpr int kRsTmaThreads = 32 * (kRsTmaConsumerWarps + 1);
constexpr int kRsTmaTile = kRsTmaConsumerWarps * 32 * 8;   // 2048 elements, one octet per consumer thread
constexpr int kRsTmaMaxStages = 8;
constexpr uint32_t kRsTmaRingBytes = 224 * 1024;           // the ring K1 keeps in flight per SM
__host__ __device__ constexpr uint32_t rs_tma_stage_bytes(int nmax) {
  return static_cast<uint32_t>(kRsTmaTile) * (2u * static_cast<uint32_t>(nmax) + 12u);
}
// As many stages as fill the ring (8 at N = 1, 4 at N = 8): bytes in flight
// per SM stay at K1's level whatever the rank count.
__host__ __device__ constexpr int rs_tma_stages(int nmax) {
  return kRsTmaRingBytes / rs_tma_stage_bytes(nmax) < kRsTmaMaxStages
             ? static_cast<int>(kRsTmaRingBytes / rs_tma_stage_bytes(nmax)) : kRsTmaMaxStages;
}
__host__ __device__ constexpr uint32_t rs_tma_smem_bytes(int nmax) {
  return rs_tma_stages(nmax) * rs_tma_stage_bytes(nmax) + 3 * kRsTmaMaxStages * 8;
}
static_assert(rs_tma_smem_bytes(1) <= 227 * 1024 && rs_tma_smem_bytes(kMaxRanks) <= 227 * 1024,
              "K1-RS TMA ring must fit the opt-in shared memory");

__device__ __forceinline__ TileLoc locate_rs_tma_tile(const UpdateParams& P, uint64_t k) {
  TileLoc t{0, 0, 0};
  for (int r = 0; r < P.nr; ++r) {
    const uint64_t body = P.r[r].n & ~7ull;
    const uint64_t nt = (body + kRsTmaTile - 1) / kRsTmaTile;
    if (k < nt) {
      t.r = r;
      t.off = k * kRsTmaTile;
      t.len = static_cast<uint32_t>(body - t.off < (uint64_t)kRsTmaTile ? body - t.off : kRsTmaTile);
      return t;
    }
    k -= nt;
  }
  t.r = -1;
  return t;
}

template <int MODE, bool CLIP>
__global__ void __launch_bounds__(kRsTmaThreads, 1) adam_update_rs_tma_kernel(const __grid_constant__ RsUpdateParams Q) {
  const UpdateParams& P = Q.u;
  extern __shared__ __align__(128) uint8_t smem[];
  int nmax = 1;
  for (int r = 0; r < P.nr; ++r) nmax = Q.gp[r].n > nmax ? Q.gp[r].n : nmax;
  const uint32_t SB = rs_tma_stage_bytes(nmax);
  const int NST = rs_tma_stages(nmax);
  const uint32_t TH = static_cast<uint32_t>(nmax) * kRsTmaTile * 2u;  // theta's offset in a stage
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + NST * SB);
  uint64_t* empty = full + kRsTmaMaxStages;
  volatile uint64_t* tile_id = empty + kRsTmaMaxStages;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int st = 0; st < NST; ++st) {
      mbar_init(&full[st], 1);
      mbar_init(&empty[st], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  __syncthreads();
  uint64_t total = 0;
  for (int r = 0; r < P.nr; ++r) total += ((P.r[r].n & ~7ull) + kRsTmaTile - 1) / kRsTmaTile;

  if (warp == kRsTmaConsumerWarps) {  // producer
    if (lane == 0) {
      const bool dyn = P.tile_ctr != nullptr;
      uint64_t k = dyn ? atomicAdd(P.tile_ctr, 1ull) - P.tile_base : blockIdx.x;
      int stage = 0;
      uint32_t phase = 0;
      for (;;) {
        uint64_t kn = k;
        if (k < total) kn = dyn ? atomicAdd(P.tile_ctr, 1ull) - P.tile_base : k + gridDim.x;
        mbar_wait(&empty[stage], phase ^ 1);
        if (k >= total) {
          tile_id[stage] = ~0ull;
          mbar_arrive(&full[stage]);
          break;
        }
        tile_id[stage] = k;
        const TileLoc t = locate_rs_tma_tile(P, k);
        const RangeDesc& R = P.r[t.r];
        const GradPeers& gp = Q.gp[t.r];
        uint8_t* base = smem + stage * SB;
        mbar_expect_tx(&full[stage], t.len * (2u * static_cast<uint32_t>(gp.n) + 12u));
        for (int q = 0; q < gp.n; ++q) bulk_load(base + q * kRsTmaTile * 2, gp.g[q] + t.off, t.len * 2u, &full[stage]);
        bulk_load(base + TH, R.th + t.off, t.len * 4u, &full[stage]);
        bulk_load(base + TH + kRsTmaTile * 4, R.m + t.off, t.len * 4u, &full[stage]);
        bulk_load(base + TH + kRsTmaTile * 8, R.v + t.off, t.len * 4u, &full[stage]);
        if (++stage == NST) {
          stage = 0;
          phase ^= 1;
        }
        k = kn;
      }
    }
  } else {  // consumers
    const double coef_d = CLIP ? clip_coef_from(P.sumsq, P.max_norm, P.nonfinite_flag) : 1.0;
    const float coef_f = static_cast<float>(coef_d);
    int stage = 0, prev_stage = -1;
    uint32_t phase = 0;
    const uint32_t o = threadIdx.x;  // octet within the tile
    for (;;) {
      mbar_wait(&full[stage], phase);
      const uint64_t k = tile_id[stage];
      if (k == ~0ull) break;
      const TileLoc t = locate_rs_tma_tile(P, k);
      const RangeDesc& R = P.r[t.r];
      const GradPeers& gp = Q.gp[t.r];
      uint8_t* base = smem + stage * SB;
      if (8 * o < t.len) {
        uint4 w[kMaxRanks];
#pragma unroll
        for (int q = 0; q < kMaxRanks; ++q)
          if (q < gp.n) w[q] = *reinterpret_cast<const uint4*>(base + q * kRsTmaTile * 2 + 16 * o);
        double sd[8];
#pragma unroll
        for (int kk = 0; kk < 8; ++kk) sd[kk] = 0.0;
#pragma unroll
        for (int q = 0; q < kMaxRanks; ++q) {
          if (q < gp.n) {
            const uint32_t ws[4] = {w[q].x, w[q].y, w[q].z, w[q].w};
#pragma unroll
            for (int kk = 0; kk < 4; ++kk) {
              sd[2 * kk] = __dadd_rn(sd[2 * kk], static_cast<double>(bf16_bits_to_f32(ws[kk] & 0xFFFFu)));
              sd[2 * kk + 1] = __dadd_rn(sd[2 * kk + 1], static_cast<double>(bf16_bits_to_f32(ws[kk] >> 16)));
            }
          }
        }
        float4* th = reinterpret_cast<float4*>(base + TH) + 2 * o;
        float4* mm = reinterpret_cast<float4*>(base + TH + kRsTmaTile * 4) + 2 * o;
        float4* vv = reinterpret_cast<float4*>(base + TH + kRsTmaTile * 8) + 2 * o;
        const float4 t0 = th[0], t1 = th[1], m0 = mm[0], m1 = mm[1], v0 = vv[0], v1 = vv[1];
        float ft[8] = {t0.x, t0.y, t0.z, t0.w, t1.x, t1.y, t1.z, t1.w};
        float fm[8] = {m0.x, m0.y, m0.z, m0.w, m1.x, m1.y, m1.z, m1.w};
        float fv[8] = {v0.x, v0.y, v0.z, v0.w, v1.x, v1.y, v1.z, v1.w};
        const bool wd = R.wd_on != 0;
#pragma unroll
        for (int kk = 0; kk < 8; ++kk)
          adam_update<MODE, CLIP>(__double2float_rn(__dmul_rn(sd[kk], gp.scale)), ft[kk], fm[kk], fv[kk], P.s, wd,
                                  coef_f, coef_d);
        th[0] = make_float4(ft[0], ft[1], ft[2], ft[3]);
        th[1] = make_float4(ft[4], ft[5], ft[6], ft[7]);
        mm[0] = make_float4(fm[0], fm[1], fm[2], fm[3]);
        mm[1] = make_float4(fm[4], fm[5], fm[6], fm[7]);
        vv[0] = make_float4(fv[0], fv[1], fv[2], fv[3]);
        vv[1] = make_float4(fv[4], fv[5], fv[6], fv[7]);
        uint4 pk;
        pk.x = pack_bf16x2_rn(ft[0], ft[1]);
        pk.y = pack_bf16x2_rn(ft[2], ft[3]);
        pk.z = pack_bf16x2_rn(ft[4], ft[5]);
        pk.w = pack_bf16x2_rn(ft[6], ft[7]);
        *reinterpret_cast<uint4*>(base + 16 * o) = pk;   // over rank 0's G16 octet (read above by this thread)
        st_peers8(P.peers[t.r], t.off + 8 * o, pk);     // fused all-gather: NVLink P2P stores
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      asm volatile("bar.sync 1, %0;" ::"r"(kRsTmaConsumerWarps * 32) : "memory");
      if (threadIdx.x == 0) {
        bulk_store(R.th + t.off, base + TH, t.len * 4u);
        bulk_store(R.m + t.off, base + TH + kRsTmaTile * 4, t.len * 4u);
        bulk_store(R.v + t.off, base + TH + kRsTmaTile * 8, t.len * 4u);
        bulk_store(R.p + t.off, base, t.len * 2u);
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
        if (prev_stage >= 0) mbar_arrive(&empty[prev_stage]);
        prev_stage = stage;
      }
      if (++stage == NST) {
        stage = 0;
        phase ^= 1;
      }
    }
    if (threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    // scalar tails (< 8 elements per range), CTA 0
    for (int r = 0; r < P.nr && blockIdx.x == 0; ++r) {
      const RangeDesc& R = P.r[r];
      const GradPeers& gp = Q.gp[r];
      const uint64_t j = (R.n & ~7ull) + threadIdx.x;
      if (j < R.n) {
        float th = R.th[j], m = R.m[j], v = R.v[j];
        adam_update<MODE, CLIP>(reduce_g1(gp, j), th, m, v, P.s, R.wd_on != 0, coef_f, coef_d);
        R.th[j] = th;
        R.m[j] = m;
        R.v[j] = v;
        const uint16_t pb = static_cast<uint16_t>(pack_bf16x2_rn(th, 0.0f) & 0xFFFFu);
        R.p[j] = pb;
        const PeerDesc& pd = P.peers[r];
        for (int q = 0; q < pd.n; ++q) pd.p[q][j] = pb;
      }
    }
    if (P.any_peers) __threadfence_system();
  }
}

__device__ __forceinline__ double warp_sum(double x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  return x;
}

// Fixed-shape CTA reduction (deterministic for a given blockDim).
__device__ __forceinline__ double block_sum(double x) {
  __shared__ double sm[kThreads / 32];
  x = warp_sum(x);
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  if (l == 0) sm[w] = x;
  __syncthreads();
  double t = 0.0;
  if (w == 0) {
    t = (l < kThreads / 32) ? sm[l] : 0.0;
    t = warp_sum(t);
  }
  return t;  // valid in thread 0
}

// K2.  Per-CTA partial of sum(g^2): g^2 is exact in fp32 for a bf16 g, the
// accumulation is in double (four independent accumulators, four 16-byte
// loads in flight per thread).  One slot per CTA, no atomics: the result is
// a fixed function of the grid, so it is reproducible run to run.
__device__ __forceinline__ double sumsq8(uint4 w) {
  const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
  double d = 0.0;
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const float lo = bf16_bits_to_f32(ws[k] & 0xFFFFu), hi = bf16_bits_to_f32(ws[k] >> 16);
    d += static_cast<double>(__fmul_rn(lo, lo));
    d += static_cast<double>(__fmul_rn(hi, hi));
  }
  return d;
}

__global__ void __launch_bounds__(kThreads) grad_sumsq_kernel(const __grid_constant__ SumsqParams P) {
  const uint64_t tid = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
  double a0 = 0.0, a1 = 0.0, a2 = 0.0, a3 = 0.0;
  for (int r = 0; r < P.nr; ++r) {
    const uint4* g = reinterpret_cast<const uint4*>(P.g[r]);
    const uint64_t n = P.n[r], n8 = n >> 3;
    uint64_t i = tid;
    for (; i + 3 * stride < n8; i += 4 * stride) {
      const uint4 w0 = __ldcs(g + i), w1 = __ldcs(g + i + stride);
      const uint4 w2 = __ldcs(g + i + 2 * stride), w3 = __ldcs(g + i + 3 * stride);
      a0 += sumsq8(w0);
      a1 += sumsq8(w1);
      a2 += sumsq8(w2);
      a3 += sumsq8(w3);
    }
    for (; i < n8; i += stride) a0 += sumsq8(__ldcs(g + i));
    const uint64_t j = (n8 << 3) + tid;
    if (j < n) {
      const float x = bf16_bits_to_f32(P.g[r][j]);
      a0 += static_cast<double>(__fmul_rn(x, x));
    }
  }
  const double t = block_sum((a0 + a1) + (a2 + a3));
  if (threadIdx.x == 0) P.partials[blockIdx.x] = t;
}

// K2-RS.  Per-CTA partial of sum(g^2) of the REDUCED gradient (the fp32 g
// the update uses), for the clip with the fused reduction.
__global__ void __launch_bounds__(kThreads) grad_sumsq_rs_kernel(const __grid_constant__ RsSumsqParams P) {
  const uint64_t tid = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
  double a0 = 0.0, a1 = 0.0;
  for (int r = 0; r < P.nr; ++r) {
    const GradPeers& gp = P.gp[r];
    const uint64_t n = P.n[r], n8 = n >> 3;
    for (uint64_t i = tid; i < n8; i += stride) {
      float g[8];
      reduce_g8(gp, 8 * i, g);
#pragma unroll
      for (int k = 0; k < 8; k += 2) {
        a0 += static_cast<double>(g[k]) * static_cast<double>(g[k]);
        a1 += static_cast<double>(g[k + 1]) * static_cast<double>(g[k + 1]);
      }
    }
    const uint64_t j = (n8 << 3) + tid;
    if (j < n) {
      const double x = static_cast<double>(reduce_g1(gp, j));
      a0 += x * x;
    }
  }
  const double t = block_sum(a0 + a1);
  if (threadIdx.x == 0) P.partials[blockIdx.x] = t;
}

// P16 refresh (ratel_refresh_params): p = bf16_rne(theta) over a rank slice,
// with the same cvt.rn.bf16x2.f32 as K1's P16 store, also into every peer's
// buffer (fused all-gather).  theta may be device memory or page-locked host
// memory read in place over the link (unified addressing); 16-byte vectors.
__global__ void __launch_bounds__(kThreads) refresh_p16_kernel(const float* __restrict__ th, uint16_t* __restrict__ p,
                                                               uint64_t n, const __grid_constant__ PeerDesc pd) {
  const uint64_t tid = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
  const uint64_t n8 = n >> 3;
  for (uint64_t i = tid; i < n8; i += stride) {
    const float4 a = *reinterpret_cast<const float4*>(th + 8 * i);
    const float4 b = *(reinterpret_cast<const float4*>(th + 8 * i) + 1);
    uint4 pk;
    pk.x = pack_bf16x2_rn(a.x, a.y);
    pk.y = pack_bf16x2_rn(a.z, a.w);
    pk.z = pack_bf16x2_rn(b.x, b.y);
    pk.w = pack_bf16x2_rn(b.z, b.w);
    *reinterpret_cast<uint4*>(p + 8 * i) = pk;
    st_peers8(pd, 8 * i, pk);
  }
  const uint64_t j = (n8 << 3) + tid;
  if (j < n) {
    const uint16_t pb = static_cast<uint16_t>(pack_bf16x2_rn(th[j], 0.0f) & 0xFFFFu);
    p[j] = pb;
    for (int q = 0; q < pd.n; ++q) pd.p[q][j] = pb;
  }
  if (pd.n > 0) __threadfence_system();
}

// K3.  One CTA sums `count` partial slots in a fixed order into *out.
__global__ void __launch_bounds__(kThreads) sumsq_finalize_kernel(const double* __restrict__ partials,
                                                                 uint64_t count, double* out) {
  double acc = 0.0;
  for (uint64_t i = threadIdx.x; i < count; i += blockDim.x) acc += partials[i];
  const double t = block_sum(acc);
  if (threadIdx.x == 0) *out = t;
}

}  // namespace ratel
