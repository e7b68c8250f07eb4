// mb_multicast.cu -- probe: NVLS multicast object over this process's device, multimem.red.add.f64 through the
// multicast address, readback through the unicast mapping; plus a timing of the flush of an n-double buffer.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o microbench/mb_multicast microbench/mb_multicast.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>

#define CK(x)                                                                   \
  do {                                                                          \
    CUresult r_ = (x);                                                          \
    if (r_ != CUDA_SUCCESS) {                                                   \
      const char* s_ = nullptr;                                                 \
      cuGetErrorString(r_, &s_);                                                \
      printf("FAIL %s: %d %s\n", #x, (int)r_, s_ ? s_ : "?");                   \
      return 1;                                                                 \
    }                                                                           \
  } while (0)

__global__ void k_mc_red(double* mc, const double* src, long n) {
  for (long i = blockIdx.x * (long)blockDim.x + threadIdx.x; i < n; i += (long)gridDim.x * blockDim.x)
    asm volatile("multimem.red.relaxed.sys.global.add.f64 [%0], %1;" ::"l"(mc + i), "d"(src[i]) : "memory");
}

int main() {
  CK(cuInit(0));
  CUdevice dev;
  CK(cuDeviceGet(&dev, 0));
  CUcontext ctx;
  CK(cuDevicePrimaryCtxRetain(&ctx, dev));
  CK(cuCtxSetCurrent(ctx));
  int mcs = 0;
  CK(cuDeviceGetAttribute(&mcs, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev));
  printf("multicast supported: %d\n", mcs);
  const long n = 3000000 + 6000 + 1;  // C4/C5 shared slice
  const size_t bytes = n * sizeof(double);
  CUmulticastObjectProp mp = {};
  mp.numDevices = 1;
  size_t gran = 0, sz = 0;
  CUmemGenericAllocationHandle mc;
  const CUmemAllocationHandleType types[3] = {(CUmemAllocationHandleType)0, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR,
                                              CU_MEM_HANDLE_TYPE_FABRIC};
  CUmemAllocationHandleType used = types[0];
  bool ok = false;
  for (int t = 0; t < 3 && !ok; ++t) {
    mp.handleTypes = types[t];
    mp.size = 0;
    CUresult r = cuMulticastGetGranularity(&gran, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED);
    if (r != CUDA_SUCCESS) { printf("granularity(type %d): %d\n", (int)types[t], (int)r); continue; }
    sz = (bytes + gran - 1) / gran * gran;
    mp.size = sz;
    r = cuMulticastCreate(&mc, &mp);
    printf("cuMulticastCreate(type %d, size %zu): %d\n", (int)types[t], sz, (int)r);
    if (r == CUDA_SUCCESS) { ok = true; used = types[t]; }
  }
  if (!ok) return 1;
  CK(cuMulticastAddDevice(mc, dev));
  CUmemAllocationProp ap = {};
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = dev;
  ap.requestedHandleTypes = used;
  size_t mgran = 0;
  CK(cuMemGetAllocationGranularity(&mgran, &ap, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED));
  printf("mem granularity %zu\n", mgran);
  CUmemGenericAllocationHandle mem;
  CK(cuMemCreate(&mem, sz, &ap, 0));
  CK(cuMulticastBindMem(mc, 0, mem, 0, sz, 0));
  CUdeviceptr uc = 0, mcp = 0;
  CK(cuMemAddressReserve(&uc, sz, gran, 0, 0));
  CK(cuMemMap(uc, sz, 0, mem, 0));
  CUmemAccessDesc ad = {};
  ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ad.location.id = dev;
  ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  CK(cuMemSetAccess(uc, sz, &ad, 1));
  CK(cuMemAddressReserve(&mcp, sz, gran, 0, 0));
  CK(cuMemMap(mcp, sz, 0, mc, 0));
  CK(cuMemSetAccess(mcp, sz, &ad, 1));
  double* src;
  cudaMalloc(&src, bytes);
  std::vector<double> h(n);
  for (long i = 0; i < n; ++i) h[i] = 0.5 * (double)(i % 1000) - 7.0;
  cudaMemcpy(src, h.data(), bytes, cudaMemcpyHostToDevice);
  cudaMemset((void*)uc, 0, sz);
  k_mc_red<<<148 * 8, 256>>>((double*)mcp, src, n);
  k_mc_red<<<148 * 8, 256>>>((double*)mcp, src, n);
  cudaError_t e = cudaDeviceSynchronize();
  printf("kernels: %s\n", cudaGetErrorString(e));
  std::vector<double> r(n);
  cudaMemcpy(r.data(), (void*)uc, bytes, cudaMemcpyDeviceToHost);
  long bad = 0;
  for (long i = 0; i < n; ++i) {
    const double want = 2 * h[i];
    if (r[i] != want) ++bad;
  }
  printf("readback mismatches: %ld of %ld\n", bad, n);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int v = 0; v < 1; ++v) {
    cudaEventRecord(a);
    for (int it = 0; it < 20; ++it) {
      k_mc_red<<<148 * 8, 256>>>((double*)mcp, src, n);
    }
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    printf("flush f64 of %ld doubles: %.1f us (%.1f GB/s)\n", n, 1e3 * ms / 20,
           bytes / (ms / 20 * 1e-3) / 1e9);
  }
  return 0;
}
