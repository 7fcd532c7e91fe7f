// Microbenchmark: per-SM throughput of the attention inner-loop instruction
// mix on sm_100a (MUFU.EX2, F2FP pack, FSEL, HMMA m16n8k16) alone and mixed.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/ubench_xu.bin tools/ubench_xu.cu
#include <cstdio>
#include <cstdint>
#include <cuda_fp16.h>

#define ITERS 4096

__device__ __forceinline__ float ex2(float x) {
  float y;
  asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ uint32_t pack(float a, float b) {
  uint32_t r;
  asm volatile("cvt.rn.f16x2.f32 %0, %2, %1;" : "=r"(r) : "f"(a), "f"(b));
  return r;
}

template <int MODE>
__global__ void k(float* out, long long* clk, float seed) {
  float v[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) v[i] = seed * (threadIdx.x + i) * 1e-3f - 3.f;
  uint32_t acc = 0;
  float c[4] = {0, 0, 0, 0};
  uint32_t a[4] = {0x3c003c00u, 0x3c003c00u, 0x3c003c00u, 0x3c003c00u};
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < ITERS; ++it) {
    if (MODE == 0) {  // 8 ex2
#pragma unroll
      for (int i = 0; i < 8; ++i) v[i] = ex2(v[i]) - 1.0f;
    } else if (MODE == 1) {  // 8 packs
#pragma unroll
      for (int i = 0; i < 8; ++i) acc += pack(v[i], v[(i + 1) & 7]), v[i] += 1e-7f;
    } else if (MODE == 2) {  // 8 ex2 + 4 packs (the attention ratio)
#pragma unroll
      for (int i = 0; i < 8; ++i) v[i] = ex2(v[i]) - 1.0f;
#pragma unroll
      for (int i = 0; i < 4; ++i) acc += pack(v[2 * i], v[2 * i + 1]);
    } else if (MODE == 3) {  // 8 HMMA m16n8k16 (independent accumulators would be better; 2 chains)
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        asm volatile(
            "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
            "{%0,%1,%2,%3};"
            : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
            : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(a[0]), "r"(a[1]));
      }
    } else if (MODE == 4) {  // 8 ex2 + 8 fsel-ish selects (predicated)
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        float s = (acc >> i) & 1 ? v[i] : -INFINITY;
        v[i] = ex2(s) - 1.0f;
      }
      acc += 0x9e3779b9u;
    }
  }
  long long t1 = clock64();
  float s = c[0] + c[1] + c[2] + c[3] + (float)acc;
#pragma unroll
  for (int i = 0; i < 8; ++i) s += v[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) clk[blockIdx.x] = t1 - t0;
}

int main() {
  float* out;
  long long* clk;
  cudaMalloc(&out, 148 * 2048 * 4);
  cudaMalloc(&clk, 148 * 8 * 8);
  const char* names[] = {"ex2 x8", "f16x2 pack x8", "ex2 x8 + pack x4", "HMMA16816 x4", "ex2 x8 + select x8"};
  const int ops[] = {8, 8, 8, 4, 8};
  for (int mode = 0; mode < 5; ++mode) {
    for (int warps : {8, 16, 32, 48}) {
      auto kern = mode == 0 ? k<0> : mode == 1 ? k<1> : mode == 2 ? k<2> : mode == 3 ? k<3> : k<4>;
      kern<<<148, warps * 32>>>(out, clk, 1.0f);
      cudaDeviceSynchronize();
      long long h[148];
      cudaMemcpy(h, clk, sizeof(h), cudaMemcpyDeviceToHost);
      double cyc = 0;
      for (int i = 0; i < 148; ++i) cyc += h[i];
      cyc /= 148;
      // lanes-ops per clock per SM for the counted op
      const double per_sm = (double)warps * 32 * ITERS * ops[mode] / cyc;
      printf("%-22s warps/SM %2d: %.1f thread-ops/clk/SM (%.2f cyc per warp-op per SMSP)\n", names[mode], warps,
             per_sm, 32.0 * 4 / per_sm);
    }
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
