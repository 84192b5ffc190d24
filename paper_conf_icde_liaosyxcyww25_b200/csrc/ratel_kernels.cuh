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
// __fmaf_rn/__fmul_rn/__fsqrt_rn/__fdiv_rn, so the compiler cannot contract
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
  float wd;                       // wd             (Adam-L2)
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

struct UpdateParams {
  RangeDesc r[kMaxRanges];
  int nr;
  AdamScalars s;
  const double* sumsq;   // clip: global sum of g^2 (device); unused otherwise
  double max_norm;
  int* nonfinite_flag;   // clip: set to !isfinite(sumsq) by CTA 0
};

struct SumsqParams {
  const uint16_t* g[kMaxRanges];
  uint64_t n[kMaxRanges];
  int nr;
  double* partials;  // one slot per CTA
};

// The per-element update.  Explicit-rounding intrinsics fix the operation
// sequence (no contraction freedom):
//   AdamW:   theta = theta*decay            (wd_on)
//   Adam-L2: g     = fma(wd, theta, g)      (wd_on)
//   m     = fma(b1, m, (1-b1)*g)
//   v     = fma(b2, v, (1-b2)*(g*g))        g*g is exact for a bf16 g
//   denom = fma(sqrt(v), 1/sqrt(bc2), eps)  == sqrt(v/bc2) + eps
//   theta = fma(-lr/bc1, m/denom, theta)
template <int MODE>
__device__ __forceinline__ void adam_update(float g, float& th, float& m, float& v,
                                            const AdamScalars& s, bool wd_on) {
  if (MODE == RATEL_ADAM_L2) {
    if (wd_on) g = __fmaf_rn(s.wd, th, g);
  } else {
    if (wd_on) th = __fmul_rn(th, s.decay);
  }
  m = __fmaf_rn(s.beta1, m, __fmul_rn(s.one_minus_beta1, g));
  v = __fmaf_rn(s.beta2, v, __fmul_rn(s.one_minus_beta2, __fmul_rn(g, g)));
  const float denom = __fmaf_rn(__fsqrt_rn(v), s.inv_sqrt_bc2, s.eps);
  th = __fmaf_rn(s.neg_step_size, __fdiv_rn(m, denom), th);
}

// 8 consecutive elements: 1x16 B of g, 2x16 B each of theta, m, v.
struct Frag8 {
  uint4 g;
  float4 t0, t1, m0, m1, v0, v1;
};

__device__ __forceinline__ void load8(Frag8& f, const RangeDesc& R, uint64_t i) {
  f.g = __ldcs(reinterpret_cast<const uint4*>(R.g) + i);
  const float4* th = reinterpret_cast<const float4*>(R.th) + 2 * i;
  const float4* m = reinterpret_cast<const float4*>(R.m) + 2 * i;
  const float4* v = reinterpret_cast<const float4*>(R.v) + 2 * i;
  f.t0 = __ldcs(th);
  f.t1 = __ldcs(th + 1);
  f.m0 = __ldcs(m);
  f.m1 = __ldcs(m + 1);
  f.v0 = __ldcs(v);
  f.v1 = __ldcs(v + 1);
}

template <int MODE, bool CLIP>
__device__ __forceinline__ void update_store8(Frag8& f, const RangeDesc& R, uint64_t i,
                                              const AdamScalars& s, float coef) {
  const uint32_t gw[4] = {f.g.x, f.g.y, f.g.z, f.g.w};
  float tt[8] = {f.t0.x, f.t0.y, f.t0.z, f.t0.w, f.t1.x, f.t1.y, f.t1.z, f.t1.w};
  float mm[8] = {f.m0.x, f.m0.y, f.m0.z, f.m0.w, f.m1.x, f.m1.y, f.m1.z, f.m1.w};
  float vv[8] = {f.v0.x, f.v0.y, f.v0.z, f.v0.w, f.v1.x, f.v1.y, f.v1.z, f.v1.w};
  const bool wd = R.wd_on != 0;
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    const uint32_t w = gw[k >> 1];
    float g = bf16_bits_to_f32((k & 1) ? (w >> 16) : (w & 0xFFFFu));
    if (CLIP) g = __fmul_rn(g, coef);
    adam_update<MODE>(g, tt[k], mm[k], vv[k], s, wd);
  }
  float4* th = reinterpret_cast<float4*>(R.th) + 2 * i;
  float4* mp = reinterpret_cast<float4*>(R.m) + 2 * i;
  float4* vp = reinterpret_cast<float4*>(R.v) + 2 * i;
  __stcs(th, make_float4(tt[0], tt[1], tt[2], tt[3]));
  __stcs(th + 1, make_float4(tt[4], tt[5], tt[6], tt[7]));
  __stcs(mp, make_float4(mm[0], mm[1], mm[2], mm[3]));
  __stcs(mp + 1, make_float4(mm[4], mm[5], mm[6], mm[7]));
  __stcs(vp, make_float4(vv[0], vv[1], vv[2], vv[3]));
  __stcs(vp + 1, make_float4(vv[4], vv[5], vv[6], vv[7]));
  uint4 pk;
  pk.x = pack_bf16x2_rn(tt[0], tt[1]);
  pk.y = pack_bf16x2_rn(tt[2], tt[3]);
  pk.z = pack_bf16x2_rn(tt[4], tt[5]);
  pk.w = pack_bf16x2_rn(tt[6], tt[7]);
  __stcs(reinterpret_cast<uint4*>(R.p) + i, pk);
}

template <int MODE, bool CLIP>
__device__ __forceinline__ void update_scalar(const RangeDesc& R, uint64_t j, const AdamScalars& s,
                                              float coef) {
  float g = bf16_bits_to_f32(R.g[j]);
  if (CLIP) g = __fmul_rn(g, coef);
  float th = R.th[j], m = R.m[j], v = R.v[j];
  adam_update<MODE>(g, th, m, v, s, R.wd_on != 0);
  R.th[j] = th;
  R.m[j] = m;
  R.v[j] = v;
  R.p[j] = static_cast<uint16_t>(pack_bf16x2_rn(th, 0.0f) & 0xFFFFu);
}

__device__ __forceinline__ float clip_coef_from(const double* sumsq, double max_norm, int* flag) {
  const double S = *sumsq;
  double c = max_norm / (sqrt(S) + 1e-6);
  c = (c < 1.0 || isnan(c)) ? c : 1.0;  // torch: clamp(max=1), NaN propagates
  if (flag != nullptr && blockIdx.x == 0 && threadIdx.x == 0) *flag = isfinite(S) ? 0 : 1;
  return static_cast<float>(c);
}

// K1.  Grid-stride over 8-element vectors of each range, 2 vectors in flight
// per thread per iteration (all 14 loads issued before any math), then the
// < 8-element scalar tail.
template <int MODE, bool CLIP>
__global__ void __launch_bounds__(kThreads) adam_update_kernel(const __grid_constant__ UpdateParams P) {
  float coef = 1.0f;
  if (CLIP) coef = clip_coef_from(P.sumsq, P.max_norm, P.nonfinite_flag);
  const uint64_t tid = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
  for (int r = 0; r < P.nr; ++r) {
    const RangeDesc R = P.r[r];
    const uint64_t n8 = R.n >> 3;
    uint64_t i = tid;
    for (; i + stride < n8; i += 2 * stride) {
      Frag8 a, b;
      load8(a, R, i);
      load8(b, R, i + stride);
      update_store8<MODE, CLIP>(a, R, i, P.s, coef);
      update_store8<MODE, CLIP>(b, R, i + stride, P.s, coef);
    }
    if (i < n8) {
      Frag8 a;
      load8(a, R, i);
      update_store8<MODE, CLIP>(a, R, i, P.s, coef);
    }
    const uint64_t j = (n8 << 3) + tid;
    if (j < R.n) update_scalar<MODE, CLIP>(R, j, P.s, coef);
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
// accumulation is in double.  One slot per CTA, no atomics.
__global__ void __launch_bounds__(kThreads) grad_sumsq_kernel(const __grid_constant__ SumsqParams P) {
  const uint64_t tid = static_cast<uint64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t stride = static_cast<uint64_t>(gridDim.x) * blockDim.x;
  double acc = 0.0;
  for (int r = 0; r < P.nr; ++r) {
    const uint16_t* g = P.g[r];
    const uint64_t n = P.n[r], n8 = n >> 3;
    for (uint64_t i = tid; i < n8; i += stride) {
      const uint4 w = __ldcs(reinterpret_cast<const uint4*>(g) + i);
      const uint32_t ws[4] = {w.x, w.y, w.z, w.w};
      double d = 0.0;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const float lo = bf16_bits_to_f32(ws[k] & 0xFFFFu), hi = bf16_bits_to_f32(ws[k] >> 16);
        d += static_cast<double>(__fmul_rn(lo, lo));
        d += static_cast<double>(__fmul_rn(hi, hi));
      }
      acc += d;
    }
    const uint64_t j = (n8 << 3) + tid;
    if (j < n) {
      const float x = bf16_bits_to_f32(g[j]);
      acc += static_cast<double>(__fmul_rn(x, x));
    }
  }
  const double t = block_sum(acc);
  if (threadIdx.x == 0) P.partials[blockIdx.x] = t;
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
