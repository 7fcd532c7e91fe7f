// Micro-benchmark: tcgen05.mma issue-to-completion cost for the small shapes
// of the attention kernel (M = 128, K = 16 per instruction, fp16 -> fp32):
// SS N = 64 (QK^T), TS N = 48 (P [V|1]), chains into ONE accumulator vs
// alternating accumulators, 1 or 2 CTAs per SM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_ipps_acharyas25_b200/csrc \
//        -I include tools/ubench_mma.cu -o /tmp/ubm && /tmp/ubm
#include <cstdio>
#include "sm100.cuh"
using namespace predtop;

template <bool TS, int N, int NACC>
__global__ void k(int iters, unsigned long long* out) {
  extern __shared__ unsigned char dsm[];
  unsigned char* base = sm100::align1024(dsm);
  __shared__ __align__(8) uint64_t bar;
  __shared__ uint32_t slot;
  const int warp = threadIdx.x / 32;
  if (threadIdx.x == 0) { sm100::mbar_init(&bar, 1); sm100::fence_mbar_init(); }
  for (int i = threadIdx.x; i < 32768 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(base)[i] = 0x3C003C00u;
  sm100::fence_proxy_async();
  if (warp == 0) sm100::tmem_alloc<256>(&slot);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem = slot;
  unsigned long long t0 = clock64();
  if (threadIdx.x == 0) {
    constexpr uint32_t id = sm100::make_idesc_f16(128, N) | (TS ? (1u << 16) : 0u);
    const uint32_t a = sm100::smem_u32(base);
    for (int it = 0; it < iters; ++it) {
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const uint32_t d = tmem + (j % NACC) * 64;
        if (TS)
          sm100::mma_f16_ts(d, tmem + 192, sm100::make_sdesc_lbo<64>(a + 1024 * (j & 3), 4096), id, 1u);
        else
          sm100::mma_f16_ss(d, sm100::make_sdesc<64>(a + 32 * (j & 1)), sm100::make_sdesc<64>(a + 8192 + 32 * (j & 1)), id, 1u);
      }
    }
    sm100::mma_commit(&bar);
    sm100::mbar_wait(&bar, 0);
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
  sm100::tc_fence_before();
  __syncthreads();
  if (warp == 0) sm100::tmem_dealloc<256>(tmem);
}

template <bool TS, int N, int NACC>
void run(const char* name, int ctas_per_sm) {
  unsigned long long* out;
  cudaMalloc(&out, 8 * 148 * 2);
  const int iters = 500;
  const int smem = 100 * 1024;
  cudaFuncSetAttribute(k<TS, N, NACC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  k<TS, N, NACC><<<148 * ctas_per_sm, 128, smem>>>(iters, out);
  cudaDeviceSynchronize();
  k<TS, N, NACC><<<148 * ctas_per_sm, 128, smem>>>(iters, out);
  cudaDeviceSynchronize();
  unsigned long long c;
  cudaMemcpy(&c, out, 8, cudaMemcpyDeviceToHost);
  printf("%-28s ctas/SM %d : %6.1f cyc per MMA (per CTA)  %s\n", name, ctas_per_sm, (double)c / (iters * 8),
         cudaGetErrorString(cudaGetLastError()));
  cudaFree(out);
}

int main() {
  for (int cps : {1, 2}) {
    run<false, 64, 1>("SS N=64 one acc", cps);
    run<false, 64, 2>("SS N=64 two accs", cps);
    run<false, 128, 1>("SS N=128 one acc", cps);
    run<false, 256, 1>("SS N=256 one acc", cps);
    run<true, 48, 1>("TS N=48 one acc", cps);
    run<true, 48, 2>("TS N=48 two accs", cps);
    run<true, 32, 1>("TS N=32 one acc", cps);
    run<true, 64, 1>("TS N=64 one acc", cps);
  }
  return 0;
}
