// Micro-benchmark: tcgen05.ld (32x32b.x16 / x32 / x64) throughput per SM as a
// function of the number of warps reading.  Build + run:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 tools/ubench_tmem.cu -o /tmp/ubt && /tmp/ubt
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ void ld16(uint32_t a, uint32_t* q) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(q[0]), "=r"(q[1]), "=r"(q[2]), "=r"(q[3]), "=r"(q[4]), "=r"(q[5]), "=r"(q[6]), "=r"(q[7]),
        "=r"(q[8]), "=r"(q[9]), "=r"(q[10]), "=r"(q[11]), "=r"(q[12]), "=r"(q[13]), "=r"(q[14]), "=r"(q[15])
      : "r"(a));
}

template <int NLD>
__global__ void k(int iters, unsigned long long* out, uint32_t* sink) {
  __shared__ uint32_t slot;
  const int warp = threadIdx.x / 32;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(
        (uint32_t)__cvta_generic_to_shared(&slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t t = slot + ((uint32_t)((warp & 3) * 32) << 16) + (warp / 4) * 64;
  uint32_t acc = 0, q[64];
  __syncthreads();
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < NLD; ++j) ld16(t + 16 * j + (it & 1) * 128, q + 16 * (j & 3));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int j = 0; j < 64; ++j) acc += q[j];
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
  sink[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(slot));
}

int main() {
  unsigned long long* out;
  uint32_t* sink;
  cudaMalloc(&out, 8 * 148);
  cudaMalloc(&sink, 4 * 148 * 1024);
  const int iters = 2000;
  for (int warps : {4, 8, 12, 16}) {
    for (int nld : {1, 2, 4}) {
      auto f = nld == 1 ? k<1> : nld == 2 ? k<2> : k<4>;
      f<<<148, warps * 32>>>(iters, out, sink);
      cudaDeviceSynchronize();
      f<<<148, warps * 32>>>(iters, out, sink);
      unsigned long long c;
      cudaMemcpy(&c, out, 8, cudaMemcpyDeviceToHost);
      double bytes = (double)iters * warps * nld * 32 * 16 * 4;
      printf("warps %2d  loads/wait %d : %8.1f B/clk/SM  (%.0f cyc per load batch per warp)\n", warps, nld,
             bytes / c, (double)c / iters);
    }
  }
  cudaError_t e = cudaGetLastError();
  printf("%s\n", cudaGetErrorString(e));
  return 0;
}
