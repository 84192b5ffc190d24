// ratel_gen.cu -- device-side synthetic inputs (harness) and test hooks.
// Same counter-based splitmix64 recipe as the host module synth/ (see
// include/ratel_gen.h); none of this is optimizer arithmetic.
#include <cuda_runtime.h>
#include <stdint.h>

#include "ratel.h"
#include "ratel_gen.h"
#include "ratel_bf16.cuh"

namespace {

constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ull;

__host__ __device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__device__ __forceinline__ uint64_t draw(uint64_t key, uint64_t i) { return mix64(key + (i + 1) * kGolden); }

__global__ void gen_theta0_kernel(float* dst, uint64_t n, uint64_t start, uint64_t key) {
  const float scale = 0.05f * 0x1p-23f;  // float32(0.05) * 2^-23, exact scaling
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t r = draw(key, start + i);
    const int32_t u = static_cast<int32_t>(r >> 40) - (1 << 23);
    dst[i] = __fmul_rn(static_cast<float>(u), scale);
  }
}

__global__ void gen_grad16_kernel(uint16_t* dst, uint64_t n, uint64_t start, uint64_t key) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t r = draw(key, start + i);
    const uint32_t sel = static_cast<uint32_t>(r >> 32) % 1000u;
    const uint32_t sign = static_cast<uint32_t>(r >> 31) & 1u;
    const uint32_t e = static_cast<uint32_t>((r >> 8) & 0xFFu) % 24u;
    const uint32_t mant = static_cast<uint32_t>(r & 0x7Fu);
    uint32_t bits = (sign << 15) | ((97u + e) << 7) | mant;
    if (sel < 10u) bits = 0x0000u;
    if (sel == 10u) bits = 0x8000u;
    dst[i] = static_cast<uint16_t>(bits);
  }
}

__global__ void bf16_rne_kernel(const float* in, uint16_t* out, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = static_cast<uint16_t>(ratel::pack_bf16x2_rn(in[i], 0.0f) & 0xFFFFu);
}

__global__ void fill_f32_kernel(float* dst, uint64_t n, float value) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x)
    dst[i] = value;
}

unsigned grid_for(uint64_t n) {
  uint64_t b = (n + 255) / 256;
  if (b > 148ull * 32) b = 148ull * 32;
  return static_cast<unsigned>(b ? b : 1);
}

int finish() {
  const cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? RATEL_OK : RATEL_ECUDA;
}

}  // namespace

extern "C" {

uint64_t ratel_gen_stream_key(uint64_t seed, uint64_t tag, uint64_t step, uint64_t block) {
  uint64_t k = mix64(seed ^ (tag * kGolden));
  k = mix64(k ^ step);
  return mix64(k ^ block);
}

int ratel_gen_theta0(float* dst, uint64_t n, uint64_t start, uint64_t key, void* stream) {
  if (n == 0) return RATEL_OK;
  if (dst == nullptr) return RATEL_EINVAL;
  gen_theta0_kernel<<<grid_for(n), 256, 0, static_cast<cudaStream_t>(stream)>>>(dst, n, start, key);
  return finish();
}

int ratel_gen_grad16(uint16_t* dst, uint64_t n, uint64_t start, uint64_t key, void* stream) {
  if (n == 0) return RATEL_OK;
  if (dst == nullptr) return RATEL_EINVAL;
  gen_grad16_kernel<<<grid_for(n), 256, 0, static_cast<cudaStream_t>(stream)>>>(dst, n, start, key);
  return finish();
}

int ratel_test_bf16_rne(const float* in, uint16_t* out, uint64_t n, void* stream) {
  if (n == 0) return RATEL_OK;
  if (in == nullptr || out == nullptr) return RATEL_EINVAL;
  bf16_rne_kernel<<<grid_for(n), 256, 0, static_cast<cudaStream_t>(stream)>>>(in, out, n);
  return finish();
}

int ratel_test_fill_f32(float* dst, uint64_t n, float value, void* stream) {
  if (n == 0) return RATEL_OK;
  if (dst == nullptr) return RATEL_EINVAL;
  fill_f32_kernel<<<grid_for(n), 256, 0, static_cast<cudaStream_t>(stream)>>>(dst, n, value);
  return finish();
}

}  // extern "C"
