// MUFU ex2 throughput: f32 vs f16x2 (results per clock per SM).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubex2 tools/ubench_ex2.cu
#include <cstdint>
#include <cstdio>
#include <cuda_fp16.h>

template <int MODE>
__global__ void k(float* out, long long* cyc, int iters) {
  float a[8];
  uint32_t h[8];
  for (int i = 0; i < 8; ++i) {
    a[i] = -0.001f * (threadIdx.x + i);
    __half2 t = __floats2half2_rn(a[i], a[i] * 0.5f);
    h[i] = *reinterpret_cast<uint32_t*>(&t);
  }
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      if (MODE == 0) {
        asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(a[i]));
      } else {
        asm volatile("ex2.approx.f16x2 %0, %0;" : "+r"(h[i]));
      }
    }
  }
  __syncthreads();
  long long t1 = clock64();
  float s = 0.f;
  for (int i = 0; i < 8; ++i) s += a[i] + __half2float(__ushort_as_half((unsigned short)h[i]));
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

int main() {
  float* out;
  long long* cyc;
  cudaMalloc(&out, 148 * 1024 * 4);
  cudaMalloc(&cyc, 148 * 8);
  const int iters = 4096;
  for (int mode = 0; mode < 2; ++mode)
    for (int threads : {128, 256, 512, 1024}) {
      long long c[148];
      for (int rep = 0; rep < 2; ++rep) {
        if (mode == 0) k<0><<<148, threads>>>(out, cyc, iters);
        else k<1><<<148, threads>>>(out, cyc, iters);
        cudaDeviceSynchronize();
      }
      cudaMemcpy(c, cyc, sizeof(c), cudaMemcpyDeviceToHost);
      const double ops = (double)threads * iters * 8 * (mode ? 2 : 1);
      printf("%s threads %4d: %.2f exp results / clk / SM (%lld cycles)\n", mode ? "f16x2" : "f32  ", threads,
             ops / c[0], c[0]);
    }
  return 0;
}
