/*
 * ratel_gen.h -- device-side synthetic input generator and test hooks.
 *
 * Harness, not the optimizer: these entry points fill device buffers with
 * the seeded synthetic inputs of DESIGN.md "Input recipe" (SURVEY §8(d)
 * "Synthetic inputs"): the same counter-based splitmix64 generator the
 * host-side module synth/ implements, so multi-GB runs on the GPU see
 * bit-identical inputs to what the CPU oracle is fed at sampled indices.
 * None of these functions touches optimizer state semantics.
 *
 * All pointers are device pointers owned by the caller; `stream` is a
 * cudaStream_t (NULL = legacy default stream).  Return 0 or a negative
 * RATEL_E* code (see ratel.h).  They do not require ratel_init.
 */
#ifndef RATEL_GEN_H
#define RATEL_GEN_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* key(seed, tag, step, block) = mix64(mix64(mix64(seed ^ tag*G) ^ step) ^ block),
 * G = 0x9E3779B97F4A7C15, mix64 = splitmix64 finaliser.  Pure host function. */
uint64_t ratel_gen_stream_key(uint64_t seed, uint64_t tag, uint64_t step, uint64_t block);

/* dst[i] = theta0 of element start+i: float32(u24 - 2^23) * float32(0.05*2^-23),
 * u24 = draw(key, start+i) >> 40.  n elements. */
int ratel_gen_theta0(float* dst, uint64_t n, uint64_t start, uint64_t key, void* stream);

/* dst[i] = bf16 gradient bits of element start+i (log-uniform magnitudes in
 * [2^-30, 2^-6), random sign, 1 % +0, 0.1 % -0). */
int ratel_gen_grad16(uint16_t* dst, uint64_t n, uint64_t start, uint64_t key, void* stream);

/* Test hook: out[i] = bf16 RNE of in[i] computed by the SAME device routine
 * the update kernel uses for P16 (cvt.rn.bf16x2.f32). n elements. */
int ratel_test_bf16_rne(const float* in, uint16_t* out, uint64_t n, void* stream);

/* Test hook: fill n fp32 elements with a constant (harness zeroing of m/v). */
int ratel_test_fill_f32(float* dst, uint64_t n, float value, void* stream);

#ifdef __cplusplus
}
#endif
#endif /* RATEL_GEN_H */
