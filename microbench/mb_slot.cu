// Microbenchmark: the fused kernel's per-item instrumental work (gather v_instr[c], then z_instr[c] += a * v-like term)
// in two shared-memory layouts, on the kernel's lane map (lane = 4 row + group j, group j's columns random in 1000).
//   A (the kernel): separate v and z arrays of doubles, bank-grouped (group j -> bank pairs 4j..4j+3);
//     ld.shared.f64 v; atomicAdd(double) z (ptxas: LDS pre-read + ATOMS.CAST.SPIN.64 loop)
//   B: interleaved 16-B (v, z) slots, bank-grouped (group j -> slot positions 2j, 2j+1 of each 128-B line);
//     one ld.shared.v2.f64 gives v and the CAS seed; explicit atom.shared.cas.b64 loop (ATOMS.CAS.64, no pre-read)
//   C: as B, slots random over the line (no grouping)
// The gap between the load and the CAS is GAP items of other work (in the kernel: one row group).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mb_slot mb_slot.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t hsh(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
  return x;
}

constexpr int kCols = 1000;      // columns per instrumental group (C3: n_instr 6000 / 6)
constexpr int kSlots = 6 * 1024; // doubles per array

template <int MODE>
__global__ void __launch_bounds__(512, 1) k(double* out, int iters) {
  extern __shared__ double sm[];  // A: v [kSlots] then z [kSlots]; B/C: (v, z) pairs [kSlots]
  for (int i = threadIdx.x; i < 2 * kSlots; i += blockDim.x) sm[i] = (MODE == 0 && i >= kSlots) ? 0.0 : 1.0;
  if (MODE != 0)
    for (int i = threadIdx.x; i < kSlots; i += blockDim.x) sm[2 * i + 1] = 0.0;
  __syncthreads();
  const int lane = threadIdx.x & 31, j = lane & 3;
  uint32_t seed = hsh(blockIdx.x * 1024 + threadIdx.x);
  double acc = 0.0;
  for (int it = 0; it < iters; ++it) {
    seed = hsh(seed + it);
    const int t = seed % kCols;
    if (MODE == 0) {
      const int slot = 16 * (t >> 2) + 4 * j + (t & 3);
      const double v = sm[slot];
      atomicAdd(sm + kSlots + slot, v);
      acc += v;
    } else {
      const int slot = MODE == 1 ? 8 * (t >> 1) + 2 * j + (t & 1) : (int)(hsh(seed) % (4 * kCols));
      double2 p;
      const uint32_t a = (uint32_t)__cvta_generic_to_shared(sm + 2 * slot);
      asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(p.x), "=d"(p.y) : "r"(a));
      unsigned long long old = __double_as_longlong(p.y), assumed;
      do {
        assumed = old;
        const unsigned long long nv = __double_as_longlong(__longlong_as_double(assumed) + p.x);
        asm volatile("atom.shared.cas.b64 %0, [%1], %2, %3;" : "=l"(old) : "r"(a + 8), "l"(assumed), "l"(nv) : "memory");
      } while (old != assumed);
      acc += p.x;
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = sm[kSlots + 1] + acc;
}

template <int MODE>
float run(double* out, int iters) {
  auto f = k<MODE>;
  const int smem = 2 * kSlots * 8 + 1024;
  cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  f<<<148, 512, smem>>>(out, 10);
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  f<<<148, 512, smem>>>(out, iters);
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
  const char* names[] = {"A: v, z arrays; atomicAdd", "B: (v,z) slots grouped; CAS", "C: (v,z) slots random; CAS"};
  float t[3] = {run<0>(out, iters), run<1>(out, iters), run<2>(out, iters)};
  for (int m = 0; m < 3; ++m)
    printf("%-32s %.3e items/s (%.2f items/SM-cycle @1.9GHz)\n", names[m], ops / (t[m] * 1e-3),
           ops / (t[m] * 1e-3) / 148 / 1.9e9);
  return cudaGetLastError() != cudaSuccess;
}
