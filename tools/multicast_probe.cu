// multicast_probe.cu -- can this box run the multimem (NVLS) form of SURVEY NEXT N1?
// N1 names `multimem.ld_reduce` / `multimem.st` on a CUDA multicast object as the
// B200-native way to fold the reduce-scatter and all-gather into the update kernel.
// The library's K1-RS uses NVLink P2P loads/stores instead; this probe records
// whether multicast objects exist here at all:
//   1. CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED on device 0;
//   2. cuMulticastCreate(numDevices = 1) + cuMulticastAddDevice + bind + map;
//   3. a kernel doing multimem.ld_reduce.add.f32 and multimem.st.f32 through the
//      mapping, checked against the unicast buffer.
// Prints one JSON line; every failing step is reported, never fatal.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o build/multicast_probe tools/multicast_probe.cu -lcuda
#include <cstdio>
#include <cstdint>
#include <cuda.h>
#include <cuda_runtime.h>

__global__ void mm_kernel(float* mc, float* out, int n) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  float v;
  asm volatile("multimem.ld_reduce.relaxed.sys.global.add.f32 %0, [%1];" : "=f"(v) : "l"(mc + i) : "memory");
  out[i] = v;
  asm volatile("multimem.st.relaxed.sys.global.f32 [%0], %1;" ::"l"(mc + i), "f"(2.f * v) : "memory");
}

static const char* errs(CUresult r) {
  const char* s = nullptr;
  cuGetErrorString(r, &s);
  return s ? s : "?";
}

int main() {
  cuInit(0);
  cudaFree(0);
  CUdevice dev;
  cuDeviceGet(&dev, 0);
  int mc_supported = -1, fabric = -1, ndev = 0;
  cuDeviceGetAttribute(&mc_supported, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev);
  cuDeviceGetAttribute(&fabric, CU_DEVICE_ATTRIBUTE_HANDLE_TYPE_FABRIC_SUPPORTED, dev);
  cudaGetDeviceCount(&ndev);
  printf("{\"devices\": %d, \"multicast_supported\": %d, \"fabric_handle_supported\": %d", ndev, mc_supported, fabric);

  const int n = 1 << 20;
  const size_t bytes = n * sizeof(float);
  // handle types to try: the create call rejects some on some systems
  const CUmemAllocationHandleType kinds[3] = {CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, CU_MEM_HANDLE_TYPE_FABRIC,
                                              CU_MEM_HANDLE_TYPE_NONE};
  const char* kname[3] = {"posix_fd", "fabric", "none"};
  CUmulticastObjectProp prop = {};
  CUmemGenericAllocationHandle mch;
  size_t gran = 0;
  CUresult r = CUDA_ERROR_UNKNOWN;
  int kind = -1;
  for (int k = 0; k < 3 && r != CUDA_SUCCESS; ++k) {
    prop = {};
    prop.numDevices = 1;
    prop.size = bytes;
    prop.handleTypes = kinds[k];
    size_t gmin = 0;
    CUresult rg = cuMulticastGetGranularity(&gmin, &prop, CU_MULTICAST_GRANULARITY_MINIMUM);
    cuMulticastGetGranularity(&gran, &prop, CU_MULTICAST_GRANULARITY_RECOMMENDED);
    printf(", \"%s_granularity\": \"%s\", \"%s_gran_min\": %zu, \"%s_gran_rec\": %zu", kname[k], errs(rg), kname[k],
           gmin, kname[k], gran);
    if (rg != CUDA_SUCCESS || gmin == 0) continue;
    gran = gmin;
    prop.size = ((bytes + gran - 1) / gran) * gran;
    r = cuMulticastCreate(&mch, &prop);
    printf(", \"%s_create\": \"%s\"", kname[k], errs(r));
    if (r == CUDA_SUCCESS) kind = k;
  }
  if (r != CUDA_SUCCESS) {   // does the create accept a 2-device object (a multi-GPU job's shape)?
    prop.numDevices = 2;
    prop.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
    prop.size = 2097152;
    CUresult r2 = cuMulticastCreate(&mch, &prop);
    printf(", \"create_2dev\": \"%s\"}\n", errs(r2));
    return 0;
  }
  r = cuMulticastAddDevice(mch, dev);
  printf(", \"add_device\": \"%s\"", errs(r));
  if (r != CUDA_SUCCESS) { printf("}\n"); return 0; }

  CUmemAllocationProp ap = {};
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = 0;
  ap.requestedHandleTypes = kinds[kind];
  CUmemGenericAllocationHandle uh;
  r = cuMemCreate(&uh, prop.size, &ap, 0);
  printf(", \"mem_create\": \"%s\"", errs(r));
  if (r != CUDA_SUCCESS) { printf("}\n"); return 0; }
  r = cuMulticastBindMem(mch, 0, uh, 0, prop.size, 0);
  printf(", \"bind\": \"%s\"", errs(r));
  if (r != CUDA_SUCCESS) { printf("}\n"); return 0; }

  CUmemAccessDesc acc = {};
  acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  acc.location.id = 0;
  acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  CUdeviceptr uva = 0, mva = 0;
  cuMemAddressReserve(&uva, prop.size, gran, 0, 0);
  cuMemMap(uva, prop.size, 0, uh, 0);
  cuMemSetAccess(uva, prop.size, &acc, 1);
  cuMemAddressReserve(&mva, prop.size, gran, 0, 0);
  r = cuMemMap(mva, prop.size, 0, mch, 0);
  printf(", \"map_multicast\": \"%s\"", errs(r));
  if (r != CUDA_SUCCESS) { printf("}\n"); return 0; }
  cuMemSetAccess(mva, prop.size, &acc, 1);

  float* host = new float[n];
  for (int i = 0; i < n; ++i) host[i] = 0.25f * (float)(i % 977) - 3.f;
  cudaMemcpy((void*)uva, host, bytes, cudaMemcpyHostToDevice);
  float* out = nullptr;
  cudaMalloc(&out, bytes);
  mm_kernel<<<(n + 255) / 256, 256>>>((float*)mva, out, n);
  cudaError_t ce = cudaDeviceSynchronize();
  printf(", \"kernel\": \"%s\"", cudaGetErrorString(ce));
  if (ce != cudaSuccess) { printf("}\n"); return 0; }
  float* back = new float[n];
  float* red = new float[n];
  cudaMemcpy(back, (void*)uva, bytes, cudaMemcpyDeviceToHost);
  cudaMemcpy(red, out, bytes, cudaMemcpyDeviceToHost);
  long bad_red = 0, bad_st = 0;
  for (int i = 0; i < n; ++i) {
    bad_red += red[i] != host[i];
    bad_st += back[i] != 2.f * host[i];
  }
  printf(", \"ld_reduce_mismatches\": %ld, \"st_mismatches\": %ld}\n", bad_red, bad_st);
  return 0;
}
