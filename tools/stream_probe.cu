// stream_probe.cu -- same-pattern HBM ceilings for K1 (SURVEY §8(d) probe 2).
// Pure data movement, no Adam math:
//   copy2   : b = a                                  (2 streams, 1R:1W)
//   soa28   : K1's pattern, 5 read streams (g bf16, theta, m, v fp32) and
//             4 write streams (theta, m, v, p)  -- 28 B/param
//   aos28   : same bytes with theta/m/v interleaved per 8-element octet
//             (2 read + 2 write streams) -- what an AoS state layout would buy
// Grid: SMs x 4 CTAs of 256 threads, grid-stride, 256-bit accesses.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/stream_probe tools/stream_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("{\"error\": \"%s line %d\"}\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

struct F8 { float r[8]; };
__device__ __forceinline__ F8 ld8(const float* p) {
  F8 f;
  asm volatile("ld.global.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(f.r[0]), "=f"(f.r[1]), "=f"(f.r[2]), "=f"(f.r[3]), "=f"(f.r[4]), "=f"(f.r[5]), "=f"(f.r[6]), "=f"(f.r[7]) : "l"(p));
  return f;
}
__device__ __forceinline__ void st8(float* p, const F8& f) {
  asm volatile("st.global.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};"
               :: "l"(p), "f"(f.r[0]), "f"(f.r[1]), "f"(f.r[2]), "f"(f.r[3]), "f"(f.r[4]), "f"(f.r[5]), "f"(f.r[6]), "f"(f.r[7]) : "memory");
}

__global__ void copy2(const float* a, float* b, uint64_t n8) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n8; i += (uint64_t)gridDim.x * blockDim.x)
    st8(b + 8 * i, ld8(a + 8 * i));
}

__global__ void soa28(const uint4* g, float* t, float* m, float* v, uint4* p, uint64_t n8) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n8; i += (uint64_t)gridDim.x * blockDim.x) {
    uint4 gg = g[i];
    F8 a = ld8(t + 8 * i), b = ld8(m + 8 * i), c = ld8(v + 8 * i);
    a.r[0] += __uint_as_float(gg.x); b.r[0] += 1.f; c.r[0] += 1.f;
    st8(t + 8 * i, a); st8(m + 8 * i, b); st8(v + 8 * i, c);
    p[i] = make_uint4(__float_as_uint(a.r[1]), gg.y, gg.z, gg.w);
  }
}

__global__ void aos28(const uint4* g, float* s, uint4* p, uint64_t n8) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n8; i += (uint64_t)gridDim.x * blockDim.x) {
    uint4 gg = g[i];
    float* q = s + 24 * i;
    F8 a = ld8(q), b = ld8(q + 8), c = ld8(q + 16);
    a.r[0] += __uint_as_float(gg.x); b.r[0] += 1.f; c.r[0] += 1.f;
    st8(q, a); st8(q + 8, b); st8(q + 16, c);
    p[i] = make_uint4(__float_as_uint(a.r[1]), gg.y, gg.z, gg.w);
  }
}

template <typename K>
float time_ms(K launch, int reps) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  launch();
  cudaDeviceSynchronize();
  float best = 1e30f;
  for (int r = 0; r < reps; ++r) {
    cudaEventRecord(e0);
    launch();
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  return best;
}

int main() {
  const uint64_t n = 314639360ull;  // one 13B block (12h^2+13h, h=5120)
  const uint64_t n8 = n / 8;
  int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  float *t, *m, *v, *s, *a, *b; uint4 *g, *p;
  CK(cudaMalloc(&t, n * 4)); CK(cudaMalloc(&m, n * 4)); CK(cudaMalloc(&v, n * 4));
  CK(cudaMalloc(&g, n * 2)); CK(cudaMalloc(&p, n * 2)); CK(cudaMalloc(&s, n * 12));
  CK(cudaMalloc(&a, n * 14)); CK(cudaMalloc(&b, n * 14));
  cudaMemset(t, 0, n * 4); cudaMemset(m, 0, n * 4); cudaMemset(v, 0, n * 4); cudaMemset(g, 0, n * 2);
  cudaMemset(s, 0, n * 12); cudaMemset(a, 0, n * 14);
  for (int cpsm : {2, 4, 8}) {
    const unsigned grid = sms * cpsm;
    const uint64_t c8 = n * 7 / 16;  // 14n bytes = 3.5n floats = 7n/16 octets
    float ms = time_ms([&] { copy2<<<grid, 256>>>(a, b, c8); }, 10);
    printf("{\"probe\": \"copy2\", \"ctas_per_sm\": %d, \"gbs\": %.1f}\n", cpsm, 28.0 * n / (ms / 1e3) / 1e9);
    ms = time_ms([&] { soa28<<<grid, 256>>>(g, t, m, v, p, n8); }, 10);
    printf("{\"probe\": \"soa28\", \"ctas_per_sm\": %d, \"gbs\": %.1f}\n", cpsm, 28.0 * n / (ms / 1e3) / 1e9);
    ms = time_ms([&] { aos28<<<grid, 256>>>(g, s, p, n8); }, 10);
    printf("{\"probe\": \"aos28\", \"ctas_per_sm\": %d, \"gbs\": %.1f}\n", cpsm, 28.0 * n / (ms / 1e3) / 1e9);
  }
  CK(cudaGetLastError());
  return 0;
}
