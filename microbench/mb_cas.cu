// Microbenchmark: throughput of shared-memory FP64 atomicAdd (ATOMS.CAST.SPIN.64 loops on sm_100a) and FP64 loads
// for address patterns of the fused kernel's instrumental slice.  One 512-thread CTA per SM, 148 CTAs.
//   mode 0: lane i -> slot (base + i) % n        (32 distinct consecutive doubles: no bank conflicts)
//   mode 1: lane i -> random slot in [0, n)      (random, 16 bank pairs)
//   mode 2: lane (r, j) -> random slot of group j in the bank-grouped layout (4 bank pairs per group; the kernel's)
//   mode 3: as 2, with one copy per row parity (each (group, copy) owns 2 bank pairs)
//   mode 4: as 2, with one copy per row r % 4 (each (group, copy) owns 1 bank pair)
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mb_cas mb_cas.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hsh(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
  return x;
}

template <int MODE, bool ATOMIC>
__global__ void __launch_bounds__(512, 1) k(double* out, int iters) {
  extern __shared__ double z[];
  const int n = 6000;
  for (int i = threadIdx.x; i < 4 * 6016; i += blockDim.x) z[i] = 0.0;
  __syncthreads();
  const int lane = threadIdx.x & 31, j = lane & 3, r = lane >> 2;
  uint32_t seed = hsh(blockIdx.x * 1024 + threadIdx.x);
  double acc = 0.0;
  for (int it = 0; it < iters; ++it) {
    seed = hsh(seed + it);
    int slot;
    if (MODE == 0) slot = (it * 32 + lane) % n;
    else if (MODE == 1) slot = seed % n;
    else {
      const int t = seed % 1000;  // column within group j (g = 1000)
      const int base = 16 * (t >> 2) + 4 * j + (t & 3);  // 4 bank pairs per group
      if (MODE == 2) slot = base;
      else if (MODE == 3) slot = 16 * (t >> 1) + 4 * j + 2 * (r & 1) + (t & 1);  // pair 4j + 2(r&1) + (t&1)
      else slot = 16 * t + 4 * j + (r & 3);                                     // pair 4j + (r&3)
    }
    if (ATOMIC) atomicAdd(z + slot, 1.0);
    else acc += z[slot];
  }
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = z[0] + acc;
}

template <int MODE, bool ATOMIC>
float run(double* out, int iters) {
  auto f = k<MODE, ATOMIC>;
  cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 4 * 6016 * 8 + 1024);
  f<<<148, 512, 4 * 6016 * 8 + 1024>>>(out, 10);
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  f<<<148, 512, 4 * 6016 * 8 + 1024>>>(out, iters);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  return ms;
}

int main() {
  double* out;
  cudaMalloc(&out, 148 * sizeof(double));
  const int iters = 4096;
  const double ops = 148.0 * 512 * iters;
  const char* names[] = {"consecutive", "random", "bank-grouped (kernel)", "2 copies (row parity)", "4 copies (row % 4)"};
  float t[5][2];
  t[0][0] = run<0, true>(out, iters); t[0][1] = run<0, false>(out, iters);
  t[1][0] = run<1, true>(out, iters); t[1][1] = run<1, false>(out, iters);
  t[2][0] = run<2, true>(out, iters); t[2][1] = run<2, false>(out, iters);
  t[3][0] = run<3, true>(out, iters); t[3][1] = run<3, false>(out, iters);
  t[4][0] = run<4, true>(out, iters); t[4][1] = run<4, false>(out, iters);
  for (int m = 0; m < 5; ++m)
    printf("%-26s atomicAdd(double) %.3e lane-ops/s (%.2f lanes/SM-cycle @1.9GHz) | ld.shared.f64 %.3e lane-ops/s\n",
           names[m], ops / (t[m][0] * 1e-3), ops / (t[m][0] * 1e-3) / 148 / 1.9e9, ops / (t[m][1] * 1e-3));
  return cudaGetLastError() != cudaSuccess;
}
