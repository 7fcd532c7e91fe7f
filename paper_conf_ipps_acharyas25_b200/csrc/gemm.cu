// gemm.cu -- tcgen05 (5th-gen tensor core) GEMM with fused epilogues for the
// per-layer dense contractions of the DAG-Transformer layer (Fig. 4):
//   QKV projection        D = X W_qkv^T + b                  -> fp16
//   FFN-1                 D = ReLU(H W_1^T + b_1)            -> fp16
//   O-proj / FFN-2 + LN   x' = LN(resid + A W^T + b)*g + be  -> fp32 + fp16
//
// One CTA computes a 128 x BN tile: TMA streams 128 x KCH (A) and BN x KCH
// (B) fp16 tiles into a 2-stage shared-memory ring (128B/64B swizzle, the UMMA
// K-major canonical layout), one elected thread issues tcgen05.mma
// (M=128, N=BN, K=16, fp32 accumulate in TMEM), and all four warps run the
// epilogue straight out of TMEM (tcgen05.ld, thread i <-> row i).  The LN
// epilogue needs the whole row in one CTA, so it runs with BN = d.
#include <algorithm>

#include "internal.h"
#include "sm100.cuh"

namespace predtop {

namespace {

constexpr int kStages = 2;
constexpr int kThreads = 128;

template <int BN>
constexpr uint32_t tmem_cols() {
  return BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : BN <= 256 ? 256 : 512;
}

template <int BN, int KCH>
constexpr int smem_bytes() {
  return kStages * (128 * KCH * 2 + BN * KCH * 2) + 1024;
}

__device__ __forceinline__ uint32_t pack_half2(float a, float b) {
  __half2 h = __floats2half2_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}

template <int BN, int KCH, int EPI>
__global__ void __launch_bounds__(kThreads, 1)
    k_gemm(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
           GemmArgs args) {
  constexpr int SW = KCH * 2;  // swizzle bytes = row bytes of a K chunk
  constexpr int A_BYTES = 128 * KCH * 2;
  constexpr int B_BYTES = BN * KCH * 2;
  constexpr uint32_t NCOLS = tmem_cols<BN>();
  extern __shared__ unsigned char dsm[];
  unsigned char* base = (unsigned char*)(((uintptr_t)dsm + 1023) & ~(uintptr_t)1023);
  unsigned char* sA = base;
  unsigned char* sB = base + kStages * A_BYTES;
  __shared__ __align__(8) uint64_t full_bar[kStages], empty_bar[kStages], acc_bar;
  __shared__ uint32_t tmem_slot;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int m0 = blockIdx.x * 128;
  const int n0 = blockIdx.y * BN;
  const int KC = args.K / KCH;

  if (threadIdx.x == 0) {
    sm100::tma_prefetch(&tmA);
    sm100::tma_prefetch(&tmB);
    for (int s = 0; s < kStages; ++s) {
      sm100::mbar_init(&full_bar[s], 1);
      sm100::mbar_init(&empty_bar[s], 1);
    }
    sm100::mbar_init(&acc_bar, 1);
    sm100::fence_mbar_init();
  }
  if (warp == 2) sm100::tmem_alloc<NCOLS>(&tmem_slot);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem = tmem_slot;

  if (warp == 0 && lane == 0) {
    // ---- TMA producer
    for (int kc = 0; kc < KC; ++kc) {
      const int s = kc % kStages;
      if (kc >= kStages) sm100::mbar_wait(&empty_bar[s], ((kc / kStages) - 1) & 1);
      sm100::mbar_arrive_expect_tx(&full_bar[s], A_BYTES + B_BYTES);
      sm100::tma_load_2d(sA + s * A_BYTES, &tmA, &full_bar[s], kc * KCH, m0);
      sm100::tma_load_2d(sB + s * B_BYTES, &tmB, &full_bar[s], kc * KCH, n0);
    }
  } else if (warp == 1 && lane == 0) {
    // ---- MMA issuer (single thread)
    constexpr uint32_t idesc = sm100::make_idesc_f16(128, BN);
    for (int kc = 0; kc < KC; ++kc) {
      const int s = kc % kStages;
      sm100::mbar_wait(&full_bar[s], (kc / kStages) & 1);
      sm100::tc_fence_after();
      const uint32_t a0 = sm100::smem_u32(sA + s * A_BYTES);
      const uint32_t b0 = sm100::smem_u32(sB + s * B_BYTES);
#pragma unroll
      for (int kk = 0; kk < KCH / 16; ++kk) {
        const uint64_t ad = sm100::make_sdesc<SW>(a0 + kk * 32);
        const uint64_t bd = sm100::make_sdesc<SW>(b0 + kk * 32);
        sm100::mma_f16_ss(tmem, ad, bd, idesc, (kc | kk) != 0);
      }
      sm100::mma_commit(&empty_bar[s]);  // frees the smem slot when these MMAs finish
    }
    sm100::mma_commit(&acc_bar);  // accumulator complete
  }
  __syncwarp();

  // ---- epilogue: thread (warp w, lane l) owns output row m0 + 32w + l
  sm100::mbar_wait(&acc_bar, 0);
  sm100::tc_fence_after();
  const int row = m0 + warp * 32 + lane;
  const bool valid = row < args.M;
  const uint32_t t_row = tmem + ((uint32_t)(warp * 32) << 16);
  float v[16];

  if constexpr (EPI == EPI_BIAS_F16 || EPI == EPI_BIAS_RELU_F16) {
    __half* out = args.out16 + (size_t)row * args.N + n0;
#pragma unroll 1
    for (int c = 0; c < BN; c += 16) {
      sm100::tmem_ld16(t_row + c, v);
      if (valid) {
        uint32_t p[8];
#pragma unroll
        for (int j = 0; j < 16; j += 2) {
          float x0 = v[j] + __ldg(args.bias + n0 + c + j);
          float x1 = v[j + 1] + __ldg(args.bias + n0 + c + j + 1);
          if (EPI == EPI_BIAS_RELU_F16) { x0 = fmaxf(x0, 0.f); x1 = fmaxf(x1, 0.f); }
          p[j / 2] = pack_half2(x0, x1);
        }
        uint4* o = reinterpret_cast<uint4*>(out + c);
        o[0] = make_uint4(p[0], p[1], p[2], p[3]);
        o[1] = make_uint4(p[4], p[5], p[6], p[7]);
      }
    }
  } else {
    // LN(resid + acc + bias): three passes over the row (mean, variance,
    // normalise + store), re-reading TMEM and the fp32 residual each pass.
    const float* res = args.resid32 + (size_t)row * BN;
    float sum = 0.f;
#pragma unroll 1
    for (int c = 0; c < BN; c += 16) {
      sm100::tmem_ld16(t_row + c, v);
      if (valid) {
#pragma unroll
        for (int j = 0; j < 16; ++j) sum += v[j] + __ldg(args.bias + c + j) + res[c + j];
      }
    }
    const float mean = sum * (1.0f / BN);
    float sq = 0.f;
#pragma unroll 1
    for (int c = 0; c < BN; c += 16) {
      sm100::tmem_ld16(t_row + c, v);
      if (valid) {
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          const float z = v[j] + __ldg(args.bias + c + j) + res[c + j] - mean;
          sq += z * z;
        }
      }
    }
    const float rstd = rsqrtf(sq * (1.0f / BN) + args.eps);
    float* o32 = args.out32 + (size_t)row * BN;
    __half* o16 = args.out16 + (size_t)row * BN;
#pragma unroll 1
    for (int c = 0; c < BN; c += 16) {
      sm100::tmem_ld16(t_row + c, v);
      if (valid) {
        float y[16];
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          const float z = v[j] + __ldg(args.bias + c + j) + res[c + j] - mean;
          y[j] = z * rstd * __ldg(args.gamma + c + j) + __ldg(args.beta + c + j);
        }
        float4* q = reinterpret_cast<float4*>(o32 + c);
#pragma unroll
        for (int j = 0; j < 4; ++j) q[j] = make_float4(y[4 * j], y[4 * j + 1], y[4 * j + 2], y[4 * j + 3]);
        uint32_t p[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) p[j] = pack_half2(y[2 * j], y[2 * j + 1]);
        uint4* h = reinterpret_cast<uint4*>(o16 + c);
        h[0] = make_uint4(p[0], p[1], p[2], p[3]);
        h[1] = make_uint4(p[4], p[5], p[6], p[7]);
      }
    }
  }

  sm100::tc_fence_before();
  __syncthreads();
  if (warp == 2) sm100::tmem_dealloc<NCOLS>(tmem);
}

template <int BN, int KCH, int EPI>
predtop_status launch_t(const CUtensorMap* tmA, const CUtensorMap* tmB, const GemmArgs& a,
                        cudaStream_t st) {
  constexpr int smem = smem_bytes<BN, KCH>();
  PT_CUDA_TRY(cudaFuncSetAttribute(k_gemm<BN, KCH, EPI>,
                                   cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  dim3 grid((unsigned)ceil_div(a.M, 128), (unsigned)(a.N / BN));
  k_gemm<BN, KCH, EPI><<<grid, kThreads, smem, st>>>(*tmA, *tmB, a);
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

template <int BN, int KCH>
predtop_status launch_epi(int epi, const CUtensorMap* tmA, const CUtensorMap* tmB,
                          const GemmArgs& a, cudaStream_t st) {
  switch (epi) {
    case EPI_BIAS_F16: return launch_t<BN, KCH, EPI_BIAS_F16>(tmA, tmB, a, st);
    case EPI_BIAS_RELU_F16: return launch_t<BN, KCH, EPI_BIAS_RELU_F16>(tmA, tmB, a, st);
    default: return launch_t<BN, KCH, EPI_BIAS_RESID_LN>(tmA, tmB, a, st);
  }
}

template <int KCH>
predtop_status launch_bn(int bn, int epi, const CUtensorMap* tmA, const CUtensorMap* tmB,
                         const GemmArgs& a, cudaStream_t st) {
  switch (bn) {
    case 32: return launch_epi<32, KCH>(epi, tmA, tmB, a, st);
    case 64: return launch_epi<64, KCH>(epi, tmA, tmB, a, st);
    case 96: return launch_epi<96, KCH>(epi, tmA, tmB, a, st);
    case 128: return launch_epi<128, KCH>(epi, tmA, tmB, a, st);
    case 192: return launch_epi<192, KCH>(epi, tmA, tmB, a, st);
    case 256: return launch_epi<256, KCH>(epi, tmA, tmB, a, st);
    default:
      set_error("unsupported GEMM tile width %d", bn);
      return PREDTOP_ERR_UNSUPPORTED;
  }
}

}  // namespace

// Output tile width for N total columns: the widest of {256,192,128,96,64,32}
// dividing N with N/BN tiles (<= 256 keeps TMEM <= 256 columns).
int gemm_pick_bn(int N) {
  const int cands[] = {256, 192, 128, 96, 64, 32};
  for (int c : cands)
    if (N % c == 0) return c;
  return 0;
}

predtop_status gemm_launch(const CUtensorMap* tmA, const CUtensorMap* tmB, int bn, int epi,
                           const GemmArgs& a, cudaStream_t st) {
  if (a.M <= 0) return PREDTOP_OK;
  if (epi == EPI_BIAS_RESID_LN && bn != a.N) {
    set_error("LN epilogue needs the whole row in one tile (bn=%d, N=%d)", bn, a.N);
    return PREDTOP_ERR_UNSUPPORTED;
  }
  if (a.K % 64 == 0) return launch_bn<64>(bn, epi, tmA, tmB, a, st);
  if (a.K == 32) return launch_bn<32>(bn, epi, tmA, tmB, a, st);
  set_error("unsupported GEMM K=%d", a.K);
  return PREDTOP_ERR_UNSUPPORTED;
}

}  // namespace predtop
