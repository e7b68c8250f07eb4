// B200 microbenchmarks that decide the aprod2 shared-slice reduction strategy and the
// row-streaming strategy. Standalone executable, not part of the
// product library. Prints one line per case: name, ops/s or GB/s.
//
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o mb_reduce mb_reduce.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>
#include <cooperative_groups.h>
namespace cg = cooperative_groups;

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  fprintf(stderr, "CUDA %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); exit(1);} } while (0)

__device__ __forceinline__ uint64_t lcg(uint64_t x) { return x * 6364136223846793005ULL + 1442695040888963407ULL; }
__device__ __forceinline__ uint32_t rnd_idx(uint64_t x, uint32_t n) { return (uint32_t)(((x >> 32) * (uint64_t)n) >> 32); }

// ---------------------------------------------------------------- streaming reads
__global__ void k_read128(const double2* __restrict__ p, size_t n2, double* out) {
  double s = 0;
  size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  #pragma unroll 4
  for (; i < n2; i += stride) { double2 v = __ldg(p + i); s += v.x + v.y; }
  if (s == 12345.678) out[0] = s;
}
__device__ __forceinline__ void ld256(const double* p, double& a, double& b, double& c, double& d) {
  asm volatile("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];" : "=d"(a), "=d"(b), "=d"(c), "=d"(d) : "l"(p));
}
__global__ void k_read256(const double* __restrict__ p, size_t n4, double* out) {
  double s = 0;
  size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  #pragma unroll 4
  for (; i < n4; i += stride) { double a, b, c, d; ld256(p + 4 * i, a, b, c, d); s += a + b + c + d; }
  if (s == 12345.678) out[0] = s;
}
__global__ void k_copy256(const double* __restrict__ p, double* __restrict__ q, size_t n4) {
  size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  #pragma unroll 4
  for (; i < n4; i += stride) {
    double a, b, c, d; ld256(p + 4 * i, a, b, c, d);
    asm volatile("st.global.v4.f64 [%0], {%1,%2,%3,%4};" :: "l"(q + 4 * i), "d"(a), "d"(b), "d"(c), "d"(d));
  }
}

// 192-B rows, 4 lanes per row, lane p reads 16-B chunks p, p+4, p+8 (row-group of 8 rows per warp)
__global__ void k_rows_rp(const double2* __restrict__ vals, const int4* __restrict__ idx, size_t n_rows,
                          double* out) {
  int lane = threadIdx.x & 31, p = lane & 3, r = lane >> 2;
  size_t warp = ((size_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  size_t nwarps = ((size_t)gridDim.x * blockDim.x) >> 5;
  double s = 0;
  #pragma unroll 2
  for (size_t g = warp; g * 8 < n_rows; g += nwarps) {
    size_t row = g * 8 + r;
    if (row < n_rows) {
      const double2* rp = vals + row * 12;
      double2 a = __ldg(rp + p), b = __ldg(rp + p + 4), c = __ldg(rp + p + 8);
      int4 ix = __ldg(idx + row);
      s += a.x + a.y + b.x + b.y + c.x + c.y + (double)(ix.x + ix.y);
    }
  }
  if (s == 12345.678) out[0] = s;
}

// ---------------------------------------------------------------- global RED patterns
// mode 0: every lane random address; mode 1: groups of 4 lanes -> 4 consecutive doubles at random base;
// mode 2: as 1 but base aligned to 4 doubles (one 32-B sector); mode 3: 8 consecutive lanes -> 8 doubles
template <int MODE>
__global__ void k_red(double* acc, uint32_t n_acc, int iters) {
  int lane = threadIdx.x & 31;
  uint64_t x = lcg(((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) * 0x9E3779B97F4A7C15ULL + 17);
  for (int it = 0; it < iters; ++it) {
    x = lcg(x);
    uint32_t a;
    if (MODE == 0) a = rnd_idx(x, n_acc);
    else {
      int grp = (MODE == 3) ? 8 : 4;
      uint64_t xs = __shfl_sync(0xffffffffu, x, lane & ~(grp - 1));
      uint32_t base = rnd_idx(xs, n_acc - grp);
      if (MODE == 2) base &= ~3u;
      a = base + (lane & (grp - 1));
    }
    atomicAdd(acc + a, 1.0);
  }
}

// ---------------------------------------------------------------- shared-memory accumulation
// smem histogram of n_acc doubles, random updates, then flushed with global RED.
template <int MODE>
__global__ void k_smem(double* acc, uint32_t n_acc, int iters) {
  extern __shared__ double sh[];
  for (uint32_t i = threadIdx.x; i < n_acc; i += blockDim.x) sh[i] = 0;
  __syncthreads();
  uint64_t x = lcg(((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) * 0x9E3779B97F4A7C15ULL + 5);
  for (int it = 0; it < iters; ++it) {
    x = lcg(x);
    uint32_t a = rnd_idx(x, n_acc);
    if (MODE == 0) atomicAdd(sh + a, 1.0);                                   // CAS loop on sm_100a
    else if (MODE == 1) atomicAdd((unsigned long long*)(sh + a), 1ULL);      // native 64-bit int?
    else if (MODE == 2) sh[a] += 1.0;                                        // racy plain RMW (throughput only)
    else if (MODE == 3) {                                                    // red.shared::cluster.add.f64 to own CTA
      uint32_t sa = (uint32_t)__cvta_generic_to_shared(sh + a);
      asm volatile("red.shared::cluster.add.f64 [%0], %1;" :: "r"(sa), "d"(1.0) : "memory");
    } else if (MODE == 4) {                                                  // fixed-point 64-bit int smem atomic
      atomicAdd((unsigned long long*)(sh + a), (unsigned long long)x);
    }
  }
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < n_acc; i += blockDim.x) atomicAdd(acc + i, sh[i]);
}

// DSMEM: cluster of 2, each CTA sends updates to partner's smem
__global__ void __cluster_dims__(2, 1, 1) k_dsmem(double* acc, uint32_t n_acc, int iters) {
  extern __shared__ double sh[];
  cg::cluster_group cl = cg::this_cluster();
  for (uint32_t i = threadIdx.x; i < n_acc; i += blockDim.x) sh[i] = 0;
  cl.sync();
  unsigned peer = cl.block_rank() ^ 1;
  uint32_t base_local = (uint32_t)__cvta_generic_to_shared(sh);
  uint32_t base_peer;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(base_peer) : "r"(base_local), "r"(peer));
  uint64_t x = lcg(((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) * 0x9E3779B97F4A7C15ULL + 9);
  for (int it = 0; it < iters; ++it) {
    x = lcg(x);
    uint32_t a = rnd_idx(x, n_acc);
    asm volatile("red.shared::cluster.add.f64 [%0], %1;" :: "r"(base_peer + 8 * a), "d"(1.0) : "memory");
  }
  cl.sync();
  for (uint32_t i = threadIdx.x; i < n_acc; i += blockDim.x) atomicAdd(acc + i, sh[i]);
}

// bulk reduce: each warp's lane 0 issues 32-B cp.reduce.async.bulk add.f64 from smem to random global sector
__global__ void k_bulkred(double* acc, uint32_t n_acc, int iters) {
  __shared__ __align__(128) double src[32][4];
  int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  if (lane < 4) src[w][lane] = 1.0;
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncwarp();
  uint64_t x = lcg(((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) * 0x9E3779B97F4A7C15ULL + 3);
  if (lane == 0) {
    uint32_t s = (uint32_t)__cvta_generic_to_shared(&src[w][0]);
    for (int it = 0; it < iters; ++it) {
      x = lcg(x);
      uint32_t a = rnd_idx(x, n_acc / 4) * 4;
      asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f64 [%0], [%1], 32;"
                   :: "l"(acc + a), "r"(s) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      if ((it & 15) == 15) asm volatile("cp.async.bulk.wait_group.read 8;" ::: "memory");
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
}

static float time_ms(cudaEvent_t a, cudaEvent_t b) { float ms; CK(cudaEventElapsedTime(&ms, a, b)); return ms; }

int main(int argc, char** argv) {
  int dev = 0; CK(cudaSetDevice(dev));
  cudaDeviceProp pr; CK(cudaGetDeviceProperties(&pr, dev));
  int nsm = pr.multiProcessorCount;
  printf("device %s sms %d l2 %d MB smem/block optin %zu KB clock %d MHz\n", pr.name, nsm, pr.l2CacheSize >> 20,
         pr.sharedMemPerBlockOptin >> 10, pr.clockRate / 1000);
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  double* out; CK(cudaMalloc(&out, 64));

  // ---- streaming
  size_t bytes = (size_t)8 << 30;
  double* big; CK(cudaMalloc(&big, bytes)); CK(cudaMemset(big, 0, bytes));
  double* big2; CK(cudaMalloc(&big2, bytes / 2));
  for (int rep = 0; rep < 2; ++rep) {
    for (int occ : {4, 8, 16}) {
      int grid = nsm * occ;
      CK(cudaEventRecord(e0));
      k_read128<<<grid, 256>>>((const double2*)big, bytes / 16, out);
      CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
      printf("read128 grid=%d  %.1f GB/s\n", grid, bytes / time_ms(e0, e1) / 1e6);
      CK(cudaEventRecord(e0));
      k_read256<<<grid, 256>>>(big, bytes / 32, out);
      CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
      printf("read256 grid=%d  %.1f GB/s\n", grid, bytes / time_ms(e0, e1) / 1e6);
      CK(cudaEventRecord(e0));
      k_copy256<<<grid, 256>>>(big, big2, bytes / 2 / 32);
      CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
      printf("copy256 grid=%d  %.1f GB/s (r+w)\n", grid, bytes / time_ms(e0, e1) / 1e6);
      size_t nrows = bytes / 208;
      CK(cudaEventRecord(e0));
      k_rows_rp<<<grid, 256>>>((const double2*)big, (const int4*)((char*)big + nrows * 192), nrows, out);
      CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
      printf("rows_rp grid=%d  %.1f GB/s\n", grid, nrows * 208.0 / time_ms(e0, e1) / 1e6);
    }
  }
  CK(cudaFree(big)); CK(cudaFree(big2));

  // ---- global RED
  double* acc; CK(cudaMalloc(&acc, (size_t)64 << 20)); CK(cudaMemset(acc, 0, (size_t)64 << 20));
  int iters = 256;
  for (uint32_t n_acc : {6000u, 30000u, 300000u, 3000000u}) {
    for (int mode = 0; mode < 4; ++mode) {
      int grid = nsm * 8;
      for (int rep = 0; rep < 2; ++rep) {
        CK(cudaEventRecord(e0));
        if (mode == 0) k_red<0><<<grid, 256>>>(acc, n_acc, iters);
        if (mode == 1) k_red<1><<<grid, 256>>>(acc, n_acc, iters);
        if (mode == 2) k_red<2><<<grid, 256>>>(acc, n_acc, iters);
        if (mode == 3) k_red<3><<<grid, 256>>>(acc, n_acc, iters);
        CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
        double ops = (double)grid * 256 * iters;
        if (rep) printf("redg mode=%d n_acc=%u  %.3g lane-ops/s  (%.2f SM-cyc per lane-op @1.9GHz)\n", mode, n_acc,
                        ops / time_ms(e0, e1) * 1e3, nsm * 1.9e9 / (ops / time_ms(e0, e1) * 1e3));
      }
    }
  }
  // ---- shared memory accumulation
  for (uint32_t n_acc : {6000u, 24000u}) {
    size_t sm = n_acc * 8;
    for (int mode = 0; mode < 5; ++mode) {
      int grid = nsm * 1, threads = 1024;
      void (*fn)(double*, uint32_t, int) = mode == 0 ? k_smem<0> : mode == 1 ? k_smem<1> : mode == 2 ? k_smem<2>
                                          : mode == 3 ? k_smem<3> : k_smem<4>;
      CK(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
      for (int rep = 0; rep < 2; ++rep) {
        CK(cudaEventRecord(e0));
        fn<<<grid, threads, sm>>>(acc, n_acc, 1024);
        CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
        cudaError_t le = cudaGetLastError();
        double ops = (double)grid * threads * 1024;
        if (rep) printf("smem mode=%d n_acc=%u  %.3g lane-ops/s  (%.2f SM-cyc per lane-op) %s\n", mode, n_acc,
                        ops / time_ms(e0, e1) * 1e3, nsm * 1.9e9 / (ops / time_ms(e0, e1) * 1e3),
                        le == cudaSuccess ? "" : cudaGetErrorString(le));
      }
    }
    {
      CK(cudaFuncSetAttribute(k_dsmem, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
      int grid = nsm, threads = 1024;
      for (int rep = 0; rep < 2; ++rep) {
        CK(cudaEventRecord(e0));
        k_dsmem<<<grid, threads, sm>>>(acc, n_acc, 1024);
        CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
        cudaError_t le = cudaGetLastError();
        double ops = (double)grid * threads * 1024;
        if (rep) printf("dsmem-red n_acc=%u  %.3g lane-ops/s  (%.2f SM-cyc per lane-op) %s\n", n_acc,
                        ops / time_ms(e0, e1) * 1e3, nsm * 1.9e9 / (ops / time_ms(e0, e1) * 1e3),
                        le == cudaSuccess ? "" : cudaGetErrorString(le));
      }
    }
  }
  // ---- bulk reduce
  for (uint32_t n_acc : {30000u, 3000000u}) {
    int grid = nsm * 4, threads = 1024;
    for (int rep = 0; rep < 2; ++rep) {
      CK(cudaEventRecord(e0));
      k_bulkred<<<grid, threads>>>(acc, n_acc, 512);
      CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
      cudaError_t le = cudaGetLastError();
      double ops = (double)grid * (threads / 32) * 512;
      if (rep) printf("bulkred32B n_acc=%u  %.3g bulk-ops/s (= %.3g double-adds/s) %s\n", n_acc,
                      ops / time_ms(e0, e1) * 1e3, 4 * ops / time_ms(e0, e1) * 1e3,
                      le == cudaSuccess ? "" : cudaGetErrorString(le));
    }
  }
  CK(cudaDeviceSynchronize());
  printf("done\n");
  return 0;
}
