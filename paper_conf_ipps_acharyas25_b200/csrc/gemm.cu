// gemm.cu -- tcgen05 (5th-gen tensor core) GEMM with fused epilogues for the
// per-layer dense contractions of the DAG-Transformer layer (Fig. 4):
//   QKV projection        D = X W_qkv^T + b                  -> fp16
//   FFN-1                 D = ReLU(H W_1^T + b_1)            -> fp16
//   O-proj / FFN-2 + LN   x' = LN(resid + A W^T + b)*g + be  -> fp32 + fp16
//
// Persistent, warp-specialised kernel, one CTA per SM:
//   warp 0      TMA producer: 128 x KCH (A) and BN x KCH (B) fp16 tiles into an
//               S-stage shared-memory ring (128B/64B swizzle = the UMMA K-major
//               canonical layout)
//   warp 1      MMA issuer: one elected thread issues tcgen05.mma
//               (M=128, N=BN, K=16, fp32 accumulate) into one of TWO TMEM
//               accumulators, so tile i+1's MMAs overlap tile i's epilogue
//   warps 2..9  epilogue (two warps per TMEM lane quarter, half the columns each): tcgen05.ld (thread <-> row), bias / ReLU / residual
//               + LayerNorm in registers, swizzled staging tile in shared
//               memory, TMA bulk-tensor store (coalesced, ragged tail clipped
//               by the tensor map).  The LN epilogue TMA-loads the fp32
//               residual tile into the same staging buffer and writes the
//               result back in place.
#include <algorithm>

#include "internal.h"
#include "sm100.cuh"

namespace predtop {

namespace {

constexpr int kThreads = 320;   // 10 warps: TMA, MMA, 8 x epilogue
constexpr int kEpiThreads = 256;
constexpr int kSmemBudget = 224 * 1024;

template <int BN>
constexpr uint32_t tmem_cols2() {  // two accumulators of BN fp32 columns
  return 2 * BN <= 32 ? 32 : 2 * BN <= 64 ? 64 : 2 * BN <= 128 ? 128 : 2 * BN <= 256 ? 256 : 512;
}

template <int BN, int KCH, int EPI>
struct Cfg {
  static constexpr int A_BYTES = 128 * KCH * 2;
  static constexpr int B_BYTES = BN * KCH * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int OUT16_BOX = BN % 64 == 0 ? 64 : 32;           // f16 store box (elements)
  static constexpr int OUT32_BYTES = EPI == EPI_BIAS_RESID_LN ? 128 * BN * 4 : 0;
  // LN with a wide row (d = 256): no room for a separate fp16 staging tile next
  // to the fp32 one and a 2-stage ring; the fp16 copy is then stored directly.
  static constexpr bool F16_DIRECT =
      EPI == EPI_BIAS_RESID_LN && 128 * BN * 6 + 2 * STAGE_BYTES + 1024 > kSmemBudget;
  // bias epilogues with 32-column-aligned halves: every epilogue warp stores
  // its own [32 rows x 32 cols] boxes from a double-buffered staging tile (no
  // CTA-wide barrier, the stores of tile i drain while tile i+1 is staged)
  static constexpr bool PER_WARP = EPI != EPI_BIAS_RESID_LN && (BN / 2) % 32 == 0;
  // double-buffered only if the operand ring keeps >= 3 stages (BN = 256
  // would drop to one stage; it keeps a single staging tile)
  static constexpr bool DBUF = PER_WARP && (kSmemBudget - 2 * 128 * BN * 2 - 1024) / STAGE_BYTES >= 3;
  static constexpr int OUT16_BYTES = F16_DIRECT ? 0 : (DBUF ? 2 : 1) * 128 * BN * 2;
  static constexpr int STAGING = OUT16_BYTES + OUT32_BYTES;
  static constexpr int STAGES_FIT = (kSmemBudget - STAGING - 1024) / STAGE_BYTES;
  static constexpr int STAGES = STAGES_FIT > 4 ? 4 : STAGES_FIT;
  static constexpr int SMEM = STAGES * STAGE_BYTES + STAGING + 1024;
  static_assert(STAGES >= 1, "shared memory budget");  // 1 only for LN at d = 256
};

__device__ __forceinline__ uint32_t pack_half2(float a, float b) {
  __half2 h = __floats2half2_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}

// Byte offset of 16-byte chunk `chunk` of row `r` inside a swizzled TMA box
// whose rows are `RB` bytes (128 -> SWIZZLE_128B, 64 -> SWIZZLE_64B).
template <int RB>
__device__ __forceinline__ uint32_t swz(int r, int chunk) {
  constexpr int mask = RB == 128 ? 7 : 3;
  const uint32_t off = (uint32_t)r * RB + (uint32_t)chunk * 16;
  return off ^ (((off >> 7) & mask) << 4);
}

__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void epi_bar() {  // named barrier over the 4 epilogue warps
  asm volatile("bar.sync 1, %0;" ::"n"(kEpiThreads) : "memory");
}
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* map, const void* smem, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(sm100::smem_u32(smem)), "r"(c0), "r"(c1)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() {
  asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read_n() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
#ifndef PREDTOP_GEMM_BOXPIPE
#define PREDTOP_GEMM_BOXPIPE 1  // 0: one bulk group per tile, waited for as a whole before restaging
#endif
constexpr bool kBoxPipe = PREDTOP_GEMM_BOXPIPE;
__device__ __forceinline__ void bulk_wait_read1() {
  asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sm100::smem_u32(bar)) : "memory");
}

struct Maps {
  CUtensorMap a, b, out16, x32;  // x32: residual load + fp32 store (LN epilogue)
  CUtensorMap out16w;            // [32 cols x 32 rows] per-warp store boxes (SW64)
};

template <int BN, int KCH, int EPI>
__global__ void __launch_bounds__(kThreads, 1)
    k_gemm(const __grid_constant__ Maps maps, GemmArgs args) {
  using C = Cfg<BN, KCH, EPI>;
  constexpr int SW = KCH * 2;
  constexpr int S = C::STAGES;
  constexpr uint32_t NCOLS = tmem_cols2<BN>();
  extern __shared__ unsigned char dsm[];
  unsigned char* base = sm100::align1024(dsm);
  unsigned char* ring = base;
  unsigned char* st16 = base + S * C::STAGE_BYTES;       // f16 output staging
  unsigned char* st32 = st16 + C::OUT16_BYTES;           // fp32 residual / output staging
  __shared__ __align__(8) uint64_t full_bar[S], empty_bar[S], tfull[2], tempty[2], resid_bar;
  __shared__ uint32_t tmem_slot;
  __shared__ float red_a[2][128], red_b[2][128];  // LN row partials of the two column halves

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ntn = args.N / BN;
  const int ntiles = (int)ceil_div(args.M, 128) * ntn;
  const int KC = args.K / KCH;

  if (threadIdx.x == 0) {
    sm100::tma_prefetch(&maps.a);
    sm100::tma_prefetch(&maps.b);
    sm100::tma_prefetch(&maps.out16);
    if (EPI == EPI_BIAS_RESID_LN) sm100::tma_prefetch(&maps.x32);
    for (int s = 0; s < S; ++s) {
      sm100::mbar_init(&full_bar[s], 1);
      sm100::mbar_init(&empty_bar[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      sm100::mbar_init(&tfull[a], 1);
      sm100::mbar_init(&tempty[a], kEpiThreads);
    }
    sm100::mbar_init(&resid_bar, 1);
    sm100::fence_mbar_init();
  }
  if (warp == 1) sm100::tmem_alloc<NCOLS>(&tmem_slot);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem = tmem_slot;

  if (warp == 0) {
    if (lane == 0) {  // ---------------- TMA producer
      int it = 0;
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const int m0 = (t / ntn) * 128, n0 = (t % ntn) * BN;
        for (int kc = 0; kc < KC; ++kc, ++it) {
          const int s = it % S;
          sm100::mbar_wait(&empty_bar[s], ((it / S) & 1) ^ 1);
          unsigned char* sa = ring + s * C::STAGE_BYTES;
          sm100::mbar_arrive_expect_tx(&full_bar[s], C::STAGE_BYTES);
          sm100::tma_load_2d(sa, &maps.a, &full_bar[s], kc * KCH, m0);
          sm100::tma_load_2d(sa + C::A_BYTES, &maps.b, &full_bar[s], kc * KCH, n0);
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {  // ---------------- MMA issuer
      constexpr uint32_t idesc = sm100::make_idesc_f16(128, BN);
      int it = 0, local = 0;
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++local) {
        const int acc = local & 1;
        sm100::mbar_wait(&tempty[acc], ((local >> 1) & 1) ^ 1);
        sm100::tc_fence_after();
        const uint32_t d_tmem = tmem + (uint32_t)(acc * BN);
        for (int kc = 0; kc < KC; ++kc, ++it) {
          const int s = it % S;
          sm100::mbar_wait(&full_bar[s], (it / S) & 1);
          sm100::tc_fence_after();
          const uint32_t a0 = sm100::smem_u32(ring + s * C::STAGE_BYTES);
          const uint32_t b0 = a0 + C::A_BYTES;
#pragma unroll
          for (int kk = 0; kk < KCH / 16; ++kk)
            sm100::mma_f16_ss(d_tmem, sm100::make_sdesc<SW>(a0 + kk * 32),
                              sm100::make_sdesc<SW>(b0 + kk * 32), idesc, (kc | kk) != 0);
          sm100::mma_commit(&empty_bar[s]);
        }
        sm100::mma_commit(&tfull[acc]);
      }
    }
  } else {
    // ---------------- epilogue warps 2..9: TMEM lane quarter q = warp % 4,
    // column half `half` (two warps per quarter split the BN columns)
    const int q = warp & 3;
    const int half = (warp - 2) >> 2;
    const int r = q * 32 + lane;  // row within the tile
    const int cbeg = half * (BN / 2), cend = cbeg + BN / 2;
    const bool leader = (warp == 2 && lane == 0);
    int local = 0;
    if constexpr (C::PER_WARP) {
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++local) {
        const int m0 = (t / ntn) * 128, n0 = (t % ntn) * BN;
        const int acc = local & 1;
        unsigned char* stage = st16 + (C::DBUF ? (local & 1) * (128 * BN * 2) : 0);
        // this warp's stores of the tile that last used this staging buffer
        // (local-2 double-buffered, local-1 otherwise) have read it.  Single
        // staging buffer with kBoxPipe: every box is its own bulk group and is
        // waited for just before it is rewritten (the box stores of tile i
        // drain while tile i+1's first boxes are staged)
        if (!kBoxPipe || C::DBUF) {
          if (lane == 0) {
            if (C::DBUF) bulk_wait_read1();
            else bulk_wait_read0();
          }
          __syncwarp();
        }
        sm100::mbar_wait(&tfull[acc], (local >> 1) & 1);
        sm100::tc_fence_after();
        const uint32_t t_row = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc * BN);
        float v[16];
        constexpr bool kPipe = kBoxPipe && !C::DBUF;
        constexpr int kNB = BN / 64;  // this warp's 32-column boxes
#pragma unroll 1
        for (int c = cbeg; c < cend; c += 16) {
          if (kPipe && c % 32 == 0) {
            if (lane == 0) bulk_wait_read_n<kNB - 1>();  // this box of the previous tile has been read
            __syncwarp();
          }
          sm100::tmem_ld16(t_row + c, v);
          const float4* b4 = reinterpret_cast<const float4*>(args.bias + n0 + c);
          float bb[16];
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const float4 t4 = __ldg(b4 + k);
            bb[4 * k] = t4.x; bb[4 * k + 1] = t4.y; bb[4 * k + 2] = t4.z; bb[4 * k + 3] = t4.w;
          }
          uint32_t p[8];
          const float qs = (n0 + c < args.qcols) ? args.qscale : 1.f;
#pragma unroll
          for (int j = 0; j < 16; j += 2) {
            float x0 = (v[j] + bb[j]) * qs;
            float x1 = (v[j + 1] + bb[j + 1]) * qs;
            if (EPI == EPI_BIAS_RELU_F16) { x0 = fmaxf(x0, 0.f); x1 = fmaxf(x1, 0.f); }
            p[j / 2] = pack_half2(x0, x1);
          }
          // box c/32: [128 rows x 32 cols] fp16, 64-byte rows, SWIZZLE_64B
          unsigned char* box = stage + (c / 32) * (128 * 64);
          const int ch = (c % 32) / 8;
          *reinterpret_cast<uint4*>(box + swz<64>(r, ch)) = make_uint4(p[0], p[1], p[2], p[3]);
          *reinterpret_cast<uint4*>(box + swz<64>(r, ch + 1)) = make_uint4(p[4], p[5], p[6], p[7]);
          if (kPipe && c % 32 == 16) {  // box complete: store it as its own bulk group
            fence_proxy_async();
            __syncwarp();
            if (lane == 0) {
              tma_store_2d(&maps.out16w, stage + (c / 32) * (128 * 64) + q * 32 * 64, n0 + c - 16, m0 + 32 * q);
              bulk_commit();
            }
          }
        }
        sm100::tc_fence_before();
        mbar_arrive(&tempty[acc]);  // accumulator may be overwritten now
        if (!kPipe) {
          fence_proxy_async();  // staging writes -> visible to the TMA (async proxy)
          __syncwarp();
          if (lane == 0) {
            // rows 32q.. of each of this warp's boxes: 32 rows x 64 B, contiguous
            for (int c = cbeg; c < cend; c += 32)
              tma_store_2d(&maps.out16w, stage + (c / 32) * (128 * 64) + q * 32 * 64, n0 + c, m0 + 32 * q);
            bulk_commit();
          }
        }
      }
      if (lane == 0) bulk_wait0();
    } else
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++local) {
      const int m0 = (t / ntn) * 128, n0 = (t % ntn) * BN;
      const int acc = local & 1;
      // staging buffers free again? (previous tile's TMA stores have read them)
      if (leader) bulk_wait_read0();
      epi_bar();
      if (EPI == EPI_BIAS_RESID_LN) {
        if (leader) {
          sm100::mbar_arrive_expect_tx(&resid_bar, C::OUT32_BYTES);
#pragma unroll
          for (int b = 0; b < BN / 32; ++b)
            sm100::tma_load_2d(st32 + b * 16384, &maps.x32, &resid_bar, n0 + b * 32, m0);
        }
      }
      sm100::mbar_wait(&tfull[acc], (local >> 1) & 1);
      sm100::tc_fence_after();
      const uint32_t t_row = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc * BN);
      float v[16];
      if constexpr (EPI == EPI_BIAS_F16 || EPI == EPI_BIAS_RELU_F16) {
#pragma unroll 1
        for (int c = cbeg; c < cend; c += 16) {
          sm100::tmem_ld16(t_row + c, v);
          const float4* b4 = reinterpret_cast<const float4*>(args.bias + n0 + c);
          float bb[16];
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const float4 t4 = __ldg(b4 + k);
            bb[4 * k] = t4.x; bb[4 * k + 1] = t4.y; bb[4 * k + 2] = t4.z; bb[4 * k + 3] = t4.w;
          }
          uint32_t p[8];
          const float qs = (n0 + c < args.qcols) ? args.qscale : 1.f;
#pragma unroll
          for (int j = 0; j < 16; j += 2) {
            float x0 = (v[j] + bb[j]) * qs;
            float x1 = (v[j + 1] + bb[j + 1]) * qs;
            if (EPI == EPI_BIAS_RELU_F16) { x0 = fmaxf(x0, 0.f); x1 = fmaxf(x1, 0.f); }
            p[j / 2] = pack_half2(x0, x1);
          }
          constexpr int RB = C::OUT16_BOX * 2;
          unsigned char* box = st16 + (c / C::OUT16_BOX) * (128 * RB);
          const int ch = (c % C::OUT16_BOX) / 8;
          *reinterpret_cast<uint4*>(box + swz<RB>(r, ch)) = make_uint4(p[0], p[1], p[2], p[3]);
          *reinterpret_cast<uint4*>(box + swz<RB>(r, ch + 1)) = make_uint4(p[4], p[5], p[6], p[7]);
        }
        sm100::tc_fence_before();
        mbar_arrive(&tempty[acc]);  // accumulator may be overwritten now
      } else {
        sm100::mbar_wait(&resid_bar, local & 1);
        // pass 1: v = acc + bias + resid (written back in place), row sum
        float sum = 0.f;
#pragma unroll 1
        for (int c = cbeg; c < cend; c += 16) {
          sm100::tmem_ld16(t_row + c, v);
          unsigned char* box = st32 + (c / 32) * 16384;
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            float4* p = reinterpret_cast<float4*>(box + swz<128>(r, (c % 32) / 4 + k));
            const float4 b = __ldg(reinterpret_cast<const float4*>(args.bias + c) + k);
            float4 x = *p;
            x.x += v[4 * k + 0] + b.x;
            x.y += v[4 * k + 1] + b.y;
            x.z += v[4 * k + 2] + b.z;
            x.w += v[4 * k + 3] + b.w;
            sum += (x.x + x.y) + (x.z + x.w);
            *p = x;
          }
        }
        sm100::tc_fence_before();
        mbar_arrive(&tempty[acc]);
        red_a[half][r] = sum;
        epi_bar();
        const float mean = (red_a[0][r] + red_a[1][r]) * (1.0f / BN);
        float sq = 0.f;
#pragma unroll 4
        for (int c4 = cbeg / 4; c4 < cend / 4; ++c4) {
          const float4 x = *reinterpret_cast<const float4*>(st32 + (c4 / 8) * 16384 + swz<128>(r, c4 % 8));
          const float a = x.x - mean, b = x.y - mean, cc = x.z - mean, d = x.w - mean;
          sq += (a * a + b * b) + (cc * cc + d * d);
        }
        red_b[half][r] = sq;
        epi_bar();
        const float rstd = rsqrtf((red_b[0][r] + red_b[1][r]) * (1.0f / BN) + args.eps);
        constexpr int RB = C::OUT16_BOX * 2;
#pragma unroll 2
        for (int c8 = cbeg / 8; c8 < cend / 8; ++c8) {  // 8 columns per iteration
          float y[8];
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int c4 = 2 * c8 + h;
            float4* p = reinterpret_cast<float4*>(st32 + (c4 / 8) * 16384 + swz<128>(r, c4 % 8));
            float4 x = *p;
            const float4 gm = __ldg(reinterpret_cast<const float4*>(args.gamma) + c4);
            const float4 bt = __ldg(reinterpret_cast<const float4*>(args.beta) + c4);
            x.x = (x.x - mean) * rstd * gm.x + bt.x;
            x.y = (x.y - mean) * rstd * gm.y + bt.y;
            x.z = (x.z - mean) * rstd * gm.z + bt.z;
            x.w = (x.w - mean) * rstd * gm.w + bt.w;
            *p = x;
            y[4 * h + 0] = x.x; y[4 * h + 1] = x.y; y[4 * h + 2] = x.z; y[4 * h + 3] = x.w;
          }
          const int c = 8 * c8;
          const uint4 pk = make_uint4(pack_half2(y[0], y[1]), pack_half2(y[2], y[3]),
                                      pack_half2(y[4], y[5]), pack_half2(y[6], y[7]));
          if constexpr (C::F16_DIRECT) {
            if (m0 + r < args.M)
              *reinterpret_cast<uint4*>(args.out16 + (size_t)(m0 + r) * args.N + c) = pk;
          } else {
            unsigned char* box = st16 + (c / C::OUT16_BOX) * (128 * RB);
            *reinterpret_cast<uint4*>(box + swz<RB>(r, (c % C::OUT16_BOX) / 8)) = pk;
          }
        }
      }
      fence_proxy_async();  // staging writes -> visible to the TMA (async proxy)
      epi_bar();
      if (leader) {
        constexpr int nb16 = C::F16_DIRECT ? 0 : BN / C::OUT16_BOX;
#pragma unroll
        for (int b = 0; b < nb16; ++b)
          tma_store_2d(&maps.out16, st16 + b * (128 * C::OUT16_BOX * 2), n0 + b * C::OUT16_BOX, m0);
        if (EPI == EPI_BIAS_RESID_LN) {
#pragma unroll
          for (int b = 0; b < BN / 32; ++b) tma_store_2d(&maps.x32, st32 + b * 16384, n0 + b * 32, m0);
        }
        bulk_commit();
      }
    }
    if (leader) bulk_wait0();
  }
  __syncwarp();
  sm100::tc_fence_before();
  __syncthreads();
  if (warp == 1) sm100::tmem_dealloc<NCOLS>(tmem);
}


template <int BN, int KCH, int EPI>
predtop_status launch_t(const Maps& maps, const GemmArgs& a, cudaStream_t st) {
  using C = Cfg<BN, KCH, EPI>;
  PT_SMEM_ATTR((k_gemm<BN, KCH, EPI>), C::SMEM);
  const int g_num_sms = num_sms();
  if (!g_num_sms) return PREDTOP_ERR_CUDA;
  const int64_t tiles = ceil_div(a.M, 128) * (a.N / BN);
  const int grid = (int)std::min<int64_t>(tiles, g_num_sms);
  k_gemm<BN, KCH, EPI><<<grid, kThreads, C::SMEM, st>>>(maps, a);
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

template <int BN, int KCH>
predtop_status launch_epi(int epi, const Maps& m, const GemmArgs& a, cudaStream_t st) {
  switch (epi) {
    case EPI_BIAS_F16: return launch_t<BN, KCH, EPI_BIAS_F16>(m, a, st);
    case EPI_BIAS_RELU_F16: return launch_t<BN, KCH, EPI_BIAS_RELU_F16>(m, a, st);
    default:
      if constexpr (BN == 32 || BN == 64 || BN == 128 || BN == 256) {
        return launch_t<BN, KCH, EPI_BIAS_RESID_LN>(m, a, st);
      } else {
        set_error("LN epilogue supports d in {32, 64, 128, 256}");
        return PREDTOP_ERR_UNSUPPORTED;
      }
  }
}

template <int KCH>
predtop_status launch_bn(int bn, int epi, const Maps& m, const GemmArgs& a, cudaStream_t st) {
  switch (bn) {
    case 32: return launch_epi<32, KCH>(epi, m, a, st);
    case 64: return launch_epi<64, KCH>(epi, m, a, st);
    case 96: return launch_epi<96, KCH>(epi, m, a, st);
    case 128: return launch_epi<128, KCH>(epi, m, a, st);
    case 192: return launch_epi<192, KCH>(epi, m, a, st);
    case 256: return launch_epi<256, KCH>(epi, m, a, st);
    default:
      set_error("unsupported GEMM tile width %d", bn);
      return PREDTOP_ERR_UNSUPPORTED;
  }
}

}  // namespace

// Output tile width for N total columns: the widest of {256,192,128,96,64,32}
// dividing N (<= 256: two fp32 accumulators fit the 512 TMEM columns).
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
  Maps m;
  m.a = *tmA;
  m.b = *tmB;
  // output / residual maps over the caller's buffers
  if (!encode_tma_2d(&m.out16, a.out16, 2, a.N, a.M, bn % 64 == 0 ? 64 : 32, 128)) return PREDTOP_ERR_CUDA;
  if (epi == EPI_BIAS_RESID_LN) {
    if (a.out32 != a.resid32) {
      set_error("LN epilogue updates the residual in place (out32 must equal resid32)");
      return PREDTOP_ERR_UNSUPPORTED;
    }
    if (!encode_tma_2d(&m.x32, a.out32, 4, a.N, a.M, 32, 128)) return PREDTOP_ERR_CUDA;
  } else {
    m.x32 = m.out16;
  }
  if (epi != EPI_BIAS_RESID_LN && (bn / 2) % 32 == 0) {
    if (!encode_tma_2d(&m.out16w, a.out16, 2, a.N, a.M, 32, 32)) return PREDTOP_ERR_CUDA;
  } else {
    m.out16w = m.out16;
  }
  if (a.kch == 32 && a.K % 32 == 0) return launch_bn<32>(bn, epi, m, a, st);
  if (a.K % 64 == 0) return launch_bn<64>(bn, epi, m, a, st);
  if (a.K == 32) return launch_bn<32>(bn, epi, m, a, st);
  set_error("unsupported GEMM K=%d", a.K);
  return PREDTOP_ERR_UNSUPPORTED;
}

}  // namespace predtop
