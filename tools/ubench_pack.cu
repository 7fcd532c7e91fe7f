// Microbenchmark: does the fp32 -> f16x2 pack (F2FP) share the MUFU/XU
// pipe with ex2 on sm_100a, and what does an integer pack cost instead?
// Per thread and iteration: 32 exponentials (the softmax thread's 32 keys)
// plus the variant's packing / masking of the 16 pairs.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubpack tools/ubench_pack.cu
#include <cstdint>
#include <cstdio>

#define ITERS 2048

__device__ __forceinline__ float ex2(float x) {
  float y;
  asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ uint32_t f2fp(float a, float b) {
  uint32_t r;
  asm volatile("cvt.rn.f16x2.f32 %0, %2, %1;" : "=r"(r) : "f"(a), "f"(b));
  return r;
}
// fp16 bits of (a, b) scaled by 2^112 taken straight from the fp32 bits:
// (a >> 13) in the low half, (b << 3) & 0xffff0000 in the high half
__device__ __forceinline__ uint32_t ipack(float a, float b) {
  uint32_t lo, hi, r;
  asm volatile("shr.b32 %0, %1, 13;" : "=r"(lo) : "r"(__float_as_uint(a)));
  asm volatile("shl.b32 %0, %1, 3;" : "=r"(hi) : "r"(__float_as_uint(b)));
  asm volatile("prmt.b32 %0, %1, %2, 0x7610;" : "=r"(r) : "r"(lo), "r"(hi));
  return r;
}
__device__ __forceinline__ uint32_t mprmt(uint32_t x0, uint32_t x1, uint32_t sel) {
  uint32_t m;
  asm volatile("prmt.b32 %0, %1, %2, %3;" : "=r"(m) : "r"(x0), "r"(x1), "r"(sel));
  return m;
}

template <int MODE>
__global__ void k(uint32_t* out, long long* clk, float seed) {
  float v[32];
#pragma unroll
  for (int i = 0; i < 32; ++i) v[i] = -seed * 1e-3f * (float)((threadIdx.x + 7 * i) & 63);
  uint32_t acc = 0, w = threadIdx.x * 0x9e3779b9u;
  __syncthreads();
  long long t0 = clock64();
#pragma unroll 1
  for (int it = 0; it < ITERS; ++it) {
    float e[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) e[i] = ex2(v[i]);
    if (MODE == 0) {
#pragma unroll
      for (int i = 0; i < 32; ++i) acc ^= __float_as_uint(e[i]);
    } else if (MODE == 1 || MODE == 3) {
#pragma unroll
      for (int i = 0; i < 16; ++i) {
        uint32_t p = f2fp(e[2 * i], e[2 * i + 1]);
        if (MODE == 3) p &= mprmt(w << (i & 7), w >> (i & 7), 0xCC88u + 0x1111u * (i & 3));
        acc ^= p;
      }
    } else if (MODE == 2 || MODE == 4) {
#pragma unroll
      for (int i = 0; i < 16; ++i) {
        uint32_t p = ipack(e[2 * i], e[2 * i + 1]);
        if (MODE == 4) p &= mprmt(w << (i & 7), w >> (i & 7), 0xCC88u + 0x1111u * (i & 3));
        acc ^= p;
      }
    } else if (MODE == 5) {  // packs only (no exponentials consumed)
#pragma unroll
      for (int i = 0; i < 16; ++i) acc ^= f2fp(v[2 * i] + (float)it, v[2 * i + 1]);
    }
    // keep the inputs live and changing (one FADD per score, as the TMEM load would)
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] = __uint_as_float((__float_as_uint(v[i]) ^ (acc & 1u)));
    w += acc;
  }
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) clk[blockIdx.x] = t1 - t0;
}

int main() {
  uint32_t* out;
  long long* clk;
  cudaMalloc(&out, 148 * 2048 * 4);
  cudaMalloc(&clk, 148 * 8 * 8);
  const char* names[] = {"32 ex2", "32 ex2 + 16 F2FP", "32 ex2 + 16 int-pack", "32 ex2 + 16 (F2FP, PRMT, AND)",
                         "32 ex2 + 16 (int-pack, PRMT, AND)", "16 F2FP only"};
  for (int mode = 0; mode < 6; ++mode) {
    for (int warps : {8, 16, 32}) {
      auto kern = mode == 0 ? k<0> : mode == 1 ? k<1> : mode == 2 ? k<2> : mode == 3 ? k<3> : mode == 4 ? k<4> : k<5>;
      kern<<<148, warps * 32>>>(out, clk, 1.0f);
      cudaDeviceSynchronize();
      long long h[148];
      cudaMemcpy(h, clk, sizeof(h), cudaMemcpyDeviceToHost);
      double cyc = 0;
      for (int i = 0; i < 148; ++i) cyc += h[i];
      cyc /= 148;
      // scores (32 per thread-iteration; pairs for mode 5) per clock per SM
      const double per_sm = (double)warps * 32 * ITERS * (mode == 5 ? 16 : 32) / cyc;
      printf("%-36s warps/SM %2d: %.2f %s/clk/SM\n", names[mode], warps, per_sm, mode == 5 ? "packs" : "scores");
    }
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
