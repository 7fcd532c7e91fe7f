// layer3.cu -- K7 v3: the post-attention half of the DAG-Transformer layer
// (Fig. 4; reading R6, post-LN encoder layer of [34]),
//     h  = LN1(x + att W_o^T + b_o)
//     x' = LN2(h + ReLU(h W_1^T + b_1) W_2^T + b_2),
// with TWO 128-row tiles per CTA (one CTA per SM) that share every weight
// slice of the ring.  The v2 kernel (layer2.cu) runs one tile per CTA and two
// CTAs per SM, each streaming all 288 KB of W_o / W_1 / W_2 per tile through
// a 64 KB ring: its FFN phase is bound by that ring's TMA latency
// (tools/tail2_trace.py).  Here a 128 KB ring feeds both tiles, so each weight
// byte is fetched once per 256 rows and the ring covers four times the time.
//
// Same scheme as v2 otherwise: acc_s (TMEM [256 s, 256 s + 128)) holds the
// O-projection of tile s, then h + b_2 written back by the epilogue, onto
// which FFN-2 accumulates; FFN-1 runs in 64-unit chunks into two TMEM buffers
// per tile (acc_s + 128 + 64 b), turned in place into the fp16 ReLU output
// that FFN-2 reads from TMEM.  The residual x tiles stream through the ring
// after the O-projection slices; x' leaves by TMA through each warp's piece
// of the h tile.
//
// Roles (18 warps): warp 0 TMA producer, warp 1 MMA issuer, warps 2..17
// epilogue: tile s = (warp - 2) / 8, lane quarter q = warp % 4 (rows 32q..),
// column half g (64 columns).
#include <algorithm>

#include "internal.h"
#include "sm100.cuh"

namespace predtop {

namespace {

constexpr int D = 128;
constexpr int FC = 64;           // FFN chunk (hidden units)
constexpr int TT = 2;            // tiles per CTA
constexpr int RS = 8;            // ring slots
constexpr int SLOT = 128 * 128;  // 16 KB
constexpr int SH = 128 * D * 2;  // fp16 h tile of one tile
constexpr int kEpiWarps = 8 * TT;
constexpr int kEpi = 32 * kEpiWarps;
constexpr int kThreads = 64 + kEpi;
constexpr int PARAMS = (6 * D + 1024) * 4;
constexpr int SMEM = RS * SLOT + TT * SH + PARAMS + 1024;
constexpr uint32_t TMEM_COLS = 512;
static_assert(SMEM <= 220 * 1024, "one CTA per SM");

struct Tail3Maps {
  CUtensorMap att, x32, x16, wo, w1, w2, x32in;
};

struct Tail3Args {
  int M, dff;
  const float *bo, *g1, *be1, *b1, *b2, *g2, *be2;
  float eps;
};

__device__ __forceinline__ void tmem_st_f32x16(uint32_t taddr, const float* v) {
  uint32_t r[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) r[i] = __float_as_uint(v[i]);
  sm100::tmem_st16(taddr, r);
}

__global__ void __launch_bounds__(kThreads, 1) k_layer_tail3(const __grid_constant__ Tail3Maps mp, Tail3Args args) {
  extern __shared__ unsigned char dsm[];
  unsigned char* base = sm100::align1024(dsm);
  unsigned char* ring = base;            // RS x 16 KB
  unsigned char* sH = ring + RS * SLOT;  // TT x [2 K-slices][128 rows x 64] fp16, SW128
  float* sPar = reinterpret_cast<float*>(sH + TT * SH);
  float* p_bo = sPar;
  float* p_g1 = sPar + D;
  float* p_be1 = sPar + 2 * D;
  float* p_b2 = sPar + 3 * D;
  float* p_g2 = sPar + 4 * D;
  float* p_be2 = sPar + 5 * D;
  float* p_b1 = sPar + 6 * D;
  for (int i = threadIdx.x; i < D; i += blockDim.x) {
    p_bo[i] = args.bo[i];
    p_g1[i] = args.g1[i];
    p_be1[i] = args.be1[i];
    p_b2[i] = args.b2[i];
    p_g2[i] = args.g2[i];
    p_be2[i] = args.be2[i];
  }
  for (int i = threadIdx.x; i < args.dff; i += blockDim.x) p_b1[i] = args.b1[i];
  __shared__ __align__(8) uint64_t ring_full[RS], ring_empty[RS];
  __shared__ __align__(8) uint64_t o_full, o_empty, h_ready, out_full;
  __shared__ __align__(8) uint64_t f_full[2], p_ready[2];
  __shared__ uint32_t tmem_slot;
  __shared__ float red[2][TT][2][128];  // [statistic][tile][column half][row]

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ntiles = (int)ceil_div(args.M, 128);
  const int npairs = (ntiles + TT - 1) / TT;
  const int NJ = args.dff / FC;
  // ring slots per pair: (TT att + 1 W_o) per K-slice, TT x 4 residual slices, W_1 / W_2 chunks
  const int SPT = (TT + 1) * (D / 64) + TT * (D / 32) + 2 * NJ;

  if (threadIdx.x == 0) {
    for (int s = 0; s < RS; ++s) {
      sm100::mbar_init(&ring_full[s], 1);
      sm100::mbar_init(&ring_empty[s], 1);
    }
    uint64_t* singles[] = {&o_full, &o_empty, &h_ready, &out_full, &f_full[0], &f_full[1]};
    for (uint64_t* b : singles) sm100::mbar_init(b, 1);
    sm100::mbar_init(&p_ready[0], kEpiWarps);
    sm100::mbar_init(&p_ready[1], kEpiWarps);
    sm100::fence_mbar_init();
  }
  if (warp == 1) sm100::tmem_alloc<TMEM_COLS>(&tmem_slot);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem = tmem_slot;

  if (warp == 0) {
    if (lane == 0) {  // ------------------------------------------ TMA producer
      sm100::tma_prefetch(&mp.att);
      sm100::tma_prefetch(&mp.x32in);
      sm100::tma_prefetch(&mp.wo);
      sm100::tma_prefetch(&mp.w1);
      sm100::tma_prefetch(&mp.w2);
      int it = 0;
      auto acquire = [&]() -> int {
        const int s = it % RS;
        sm100::mbar_wait(&ring_empty[s], ((it / RS) & 1) ^ 1);
        sm100::mbar_arrive_expect_tx(&ring_full[s], SLOT);
        return s;
      };
      auto load = [&](const CUtensorMap* m, int c0, int c1) {
        const int s = acquire();
        sm100::tma_load_2d(ring + s * SLOT, m, &ring_full[s], c0, c1);
        ++it;
      };
      auto load_w1 = [&](int j) {  // [64 hidden x 128 K] as two [64 x 64] K-slices
        const int s = acquire();
        for (int kc = 0; kc < D / 64; ++kc)
          sm100::tma_load_2d(ring + s * SLOT + kc * (FC * 128), &mp.w1, &ring_full[s], kc * 64, j * FC);
        ++it;
      };
      for (int p = blockIdx.x; p < npairs; p += gridDim.x) {
        const int m0 = p * TT * 128;
        for (int kc = 0; kc < D / 64; ++kc) {
          for (int s = 0; s < TT; ++s) load(&mp.att, kc * 64, m0 + 128 * s);
          load(&mp.wo, kc * 64, 0);
        }
        for (int s = 0; s < TT; ++s)
          for (int k = 0; k < D / 32; ++k) load(&mp.x32in, k * 32, m0 + 128 * s);
        load_w1(0);
        for (int j = 0; j < NJ; ++j) {
          if (j + 1 < NJ) load_w1(j + 1);
          load(&mp.w2, j * FC, 0);
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {  // ------------------------------------------ MMA issuer
      constexpr uint32_t id_N128 = sm100::make_idesc_f16(128, 128);
      constexpr uint32_t id_N64 = sm100::make_idesc_f16(128, FC);
      int it = 0;
      auto slot_wait = [&]() -> uint32_t {
        const int s = it % RS;
        sm100::mbar_wait(&ring_full[s], (it / RS) & 1);
        sm100::tc_fence_after();
        return sm100::smem_u32(ring + s * SLOT);
      };
      const uint32_t aH = sm100::smem_u32(sH);
      int i = 0;
      for (int p = blockIdx.x; p < npairs; p += gridDim.x, ++i) {
        // ---- O-projection of both tiles (acc_s free once LN2 of the previous pair read it)
        sm100::mbar_wait(&o_empty, (i & 1) ^ 1);
        sm100::tc_fence_after();
        for (int kc = 0; kc < D / 64; ++kc) {
          uint32_t a[TT];
          int sa[TT];
          for (int s = 0; s < TT; ++s) {
            a[s] = slot_wait();
            sa[s] = it % RS;
            ++it;
          }
          const uint32_t b0 = slot_wait();
          for (int s = 0; s < TT; ++s)
#pragma unroll
            for (int kk = 0; kk < 4; ++kk)
              sm100::mma_f16_ss(tmem + 256 * s, sm100::make_sdesc<128>(a[s] + kk * 32),
                                sm100::make_sdesc<128>(b0 + kk * 32), id_N128, (kc | kk) != 0);
          for (int s = 0; s < TT; ++s) sm100::mma_commit(&ring_empty[sa[s]]);
          sm100::mma_commit(&ring_empty[it % RS]);
          ++it;
        }
        sm100::mma_commit(&o_full);
        // the x slots belong to the epilogue; the next slot_wait (FFN-1, after
        // h_ready) is on a phase whose predecessor the epilogue consumed
        it += TT * (D / 32);
        sm100::mbar_wait(&h_ready, i & 1);
        sm100::tc_fence_after();
        auto ffn1 = [&](int j) {
          const uint32_t b0 = slot_wait();
          for (int s = 0; s < TT; ++s) {
            const uint32_t dst = tmem + 256 * s + 128 + (uint32_t)((j & 1) * FC);
#pragma unroll
            for (int kc = 0; kc < D / 64; ++kc)
#pragma unroll
              for (int kk = 0; kk < 4; ++kk)
                sm100::mma_f16_ss(dst, sm100::make_sdesc<128>(aH + s * SH + kc * SLOT + kk * 32),
                                  sm100::make_sdesc<128>(b0 + kc * (FC * 128) + kk * 32), id_N64,
                                  (kc | kk) != 0);
          }
          sm100::mma_commit(&ring_empty[it % RS]);
          ++it;
          sm100::mma_commit(&f_full[j & 1]);
        };
        ffn1(0);
        for (int j = 0; j < NJ; ++j) {
          if (j + 1 < NJ) ffn1(j + 1);
          sm100::mbar_wait(&p_ready[j & 1], ((i * NJ + j) >> 1) & 1);
          sm100::tc_fence_after();
          const uint32_t b0 = slot_wait();
          for (int s = 0; s < TT; ++s) {
            const uint32_t src = tmem + 256 * s + 128 + (uint32_t)((j & 1) * FC);
#pragma unroll
            for (int ks = 0; ks < FC / 16; ++ks)
              sm100::mma_f16_ts(tmem + 256 * s, src + (uint32_t)(32 * (ks / 2) + 8 * (ks % 2)),
                                sm100::make_sdesc<128>(b0 + ks * 32), id_N128, 1u);
          }
          sm100::mma_commit(&ring_empty[it % RS]);
          ++it;
        }
        sm100::mma_commit(&out_full);
      }
    }
  } else {
    // ------------------------------------------ epilogue warps 2..17
    const int ew = warp - 2;
    const int ts = ew >> 3;                   // tile of the pair
    const int q = warp & 3, g = (ew >> 2) & 1;
    const int r = q * 32 + lane;              // tile row (TMEM lane)
    const uint32_t lrow = (uint32_t)(q * 32) << 16;
    const uint32_t acc = tmem + 256 * ts, acc_f = acc + 128;
    const bool leader = (ew == 0 && lane == 0);
    unsigned char* stg = sH + ts * SH + g * SLOT + q * 4096;  // this warp's 4 KB piece
    auto store_wait = [&]() {
      if (lane == 0) sm100::bulk_wait_read0();
      __syncwarp();
    };
    auto row_sum = [&](float s, int which) {
      red[which][ts][g][r] = s;
      sm100::named_bar<kEpi>(1);
      return red[which][ts][0][r] + red[which][ts][1][r];
    };
    float x[64];
    int i = 0;
    for (int p = blockIdx.x; p < npairs; p += gridDim.x, ++i) {
      const int m0 = (p * TT + ts) * 128;
      const int cbase = i * NJ;
      // ---- residual x from the ring (after o_full: no parity aliasing)
      sm100::mbar_wait(&o_full, i & 1);
      sm100::tc_fence_after();
      const int xit = i * SPT + (TT + 1) * (D / 64);
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        const int itk = xit + ts * (D / 32) + 2 * g + k;
        sm100::mbar_wait(&ring_full[itk % RS], (itk / RS) & 1);
        const unsigned char* sl = ring + (itk % RS) * SLOT;
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          const float4 v = *reinterpret_cast<const float4*>(sl + sm100::swz<128>(r, c));
          x[32 * k + 4 * c] = v.x;
          x[32 * k + 4 * c + 1] = v.y;
          x[32 * k + 4 * c + 2] = v.z;
          x[32 * k + 4 * c + 3] = v.w;
        }
      }
      sm100::fence_proxy_async();
      // ---- LN1: z = x + acc + b_o
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        float a[16];
        sm100::tmem_ld16(acc + lrow + 64 * g + 16 * k, a);
#pragma unroll
        for (int e = 0; e < 16; ++e) x[16 * k + e] += a[e] + p_bo[64 * g + 16 * k + e];
      }
      {
        float s = 0.f;
#pragma unroll
        for (int e = 0; e < 64; ++e) s += x[e];
        const float mean = row_sum(s, 0) * (1.0f / D);
        if (leader)  // every epilogue thread has read its x: free the x slots
          for (int k = 0; k < TT * (D / 32); ++k) sm100::mbar_arrive(&ring_empty[(xit + k) % RS]);
        float sq = 0.f;
#pragma unroll
        for (int e = 0; e < 64; ++e) {
          const float dlt = x[e] - mean;
          sq += dlt * dlt;
        }
        const float rstd = rsqrtf(row_sum(sq, 1) * (1.0f / D) + args.eps);
#pragma unroll
        for (int e = 0; e < 64; ++e) x[e] = (x[e] - mean) * rstd * p_g1[64 * g + e] + p_be1[64 * g + e];
      }
      store_wait();  // the previous pair's x16 store has read the piece
#pragma unroll
      for (int c = 0; c < 8; ++c)
        *reinterpret_cast<uint4*>(stg + sm100::swz<128>(lane, c)) =
            make_uint4(sm100::pack_half2(x[8 * c], x[8 * c + 1]), sm100::pack_half2(x[8 * c + 2], x[8 * c + 3]),
                       sm100::pack_half2(x[8 * c + 4], x[8 * c + 5]), sm100::pack_half2(x[8 * c + 6], x[8 * c + 7]));
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        float hb[16];
#pragma unroll
        for (int e = 0; e < 16; ++e) hb[e] = x[16 * k + e] + p_b2[64 * g + 16 * k + e];
        tmem_st_f32x16(acc + lrow + 64 * g + 16 * k, hb);
      }
      sm100::tmem_wait_st();
      sm100::fence_proxy_async();
      sm100::tc_fence_before();
      sm100::named_bar<kEpi>(1);
      if (leader) sm100::mbar_arrive(&h_ready);
      // ---- FFN chunks: ReLU(acc_f + b_1) -> fp16 pairs back into the buffer
      for (int j = 0; j < NJ; ++j) {
        const int cj = cbase + j;
        sm100::mbar_wait(&f_full[j & 1], (cj >> 1) & 1);
        sm100::tc_fence_after();
        {
          const uint32_t buf = acc_f + (uint32_t)((j & 1) * FC);
          float v[32];
          sm100::tmem_ld<32>(buf + lrow + 32 * g, v);
          const float* b1 = p_b1 + j * FC + 32 * g;
          uint32_t pk[16];
#pragma unroll
          for (int k = 0; k < 16; ++k)
            pk[k] = sm100::pack_half2(fmaxf(v[2 * k] + b1[2 * k], 0.f), fmaxf(v[2 * k + 1] + b1[2 * k + 1], 0.f));
          sm100::tmem_st16(buf + lrow + 32 * g, pk);
        }
        sm100::tmem_wait_st();
        sm100::tc_fence_before();
        __syncwarp();
        if (lane == 0) sm100::mbar_arrive(&p_ready[j & 1]);
      }
      // ---- LN2: z = acc (= h + b_2 + FFN(h))
      sm100::mbar_wait(&out_full, i & 1);
      sm100::tc_fence_after();
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        float a[32];
        sm100::tmem_ld<32>(acc + lrow + 64 * g + 32 * k, a);
#pragma unroll
        for (int e = 0; e < 32; ++e) x[32 * k + e] = a[e];
      }
      sm100::tc_fence_before();
      {
        float s = 0.f;
#pragma unroll
        for (int e = 0; e < 64; ++e) s += x[e];
        const float mean = row_sum(s, 0) * (1.0f / D);
        if (leader) sm100::mbar_arrive(&o_empty);  // every epilogue thread has read acc
        float sq = 0.f;
#pragma unroll
        for (int e = 0; e < 64; ++e) {
          const float dlt = x[e] - mean;
          sq += dlt * dlt;
        }
        const float rstd = rsqrtf(row_sum(sq, 1) * (1.0f / D) + args.eps);
#pragma unroll
        for (int e = 0; e < 64; ++e) x[e] = (x[e] - mean) * rstd * p_g2[64 * g + e] + p_be2[64 * g + e];
      }
      // ---- x' (fp32, two [32 x 32] boxes) and its fp16 shadow through the piece
      // (the piece held h, read by FFN-1 MMAs that completed before out_full)
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        if (k) store_wait();
#pragma unroll
        for (int c = 0; c < 8; ++c)
          *reinterpret_cast<float4*>(stg + sm100::swz<128>(lane, c)) =
              make_float4(x[32 * k + 4 * c], x[32 * k + 4 * c + 1], x[32 * k + 4 * c + 2], x[32 * k + 4 * c + 3]);
        sm100::fence_proxy_async();
        __syncwarp();
        if (lane == 0) {
          sm100::tma_store_2d(&mp.x32, stg, 64 * g + 32 * k, m0 + 32 * q);
          sm100::bulk_commit();
        }
      }
      store_wait();
#pragma unroll
      for (int c = 0; c < 8; ++c)
        *reinterpret_cast<uint4*>(stg + sm100::swz<128>(lane, c)) =
            make_uint4(sm100::pack_half2(x[8 * c], x[8 * c + 1]), sm100::pack_half2(x[8 * c + 2], x[8 * c + 3]),
                       sm100::pack_half2(x[8 * c + 4], x[8 * c + 5]), sm100::pack_half2(x[8 * c + 6], x[8 * c + 7]));
      sm100::fence_proxy_async();
      __syncwarp();
      if (lane == 0) {
        sm100::tma_store_2d(&mp.x16, stg, 64 * g, m0 + 32 * q);
        sm100::bulk_commit();
      }
    }
    if (lane == 0) sm100::bulk_wait0();
  }
  __syncwarp();
  sm100::tc_fence_before();
  __syncthreads();
  if (warp == 1) sm100::tmem_dealloc<TMEM_COLS>(tmem);
}

int g_sms3 = 0;

}  // namespace

bool layer_tail3_supported(int d, int dff) { return d == D && dff % (2 * FC) == 0 && dff <= 1024; }

predtop_status layer_tail3_launch(const predtop_model_s* m, int l, const __half* att, float* x32,
                                  __half* x16, int M, cudaStream_t st) {
  const int d = m->cfg.d_model, dff = m->cfg.d_ff;
  if (!layer_tail3_supported(d, dff)) {
    set_error("layer tail v3 needs d = 128 and d_ff %% 128 == 0");
    return PREDTOP_ERR_UNSUPPORTED;
  }
  if (M <= 0) return PREDTOP_OK;
  const LayerDev& L = m->layer[l];
  Tail3Maps mp;
  if (!encode_tma_2d(&mp.att, att, 2, d, M, 64, 128) || !encode_tma_2d(&mp.x32, x32, 4, d, M, 32, 32) ||
      !encode_tma_2d(&mp.x16, x16, 2, d, M, 64, 32) || !encode_tma_2d(&mp.x32in, x32, 4, d, M, 32, 128))
    return PREDTOP_ERR_CUDA;
  mp.wo = L.tm_o;
  mp.w1 = L.tm_1h;
  mp.w2 = L.tm_2;
  Tail3Args a{M, dff, L.bo, L.g1, L.be1, L.b1, L.b2, L.g2, L.be2, m->cfg.ln_eps};
  static bool attr_done = false;
  if (!attr_done) {
    PT_CUDA_TRY(cudaFuncSetAttribute(k_layer_tail3, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM));
    attr_done = true;
  }
  if (!g_sms3) {
    int dev = 0;
    PT_CUDA_TRY(cudaGetDevice(&dev));
    PT_CUDA_TRY(cudaDeviceGetAttribute(&g_sms3, cudaDevAttrMultiProcessorCount, dev));
  }
  const int pairs = (int)ceil_div(ceil_div(M, 128), TT);
  const int grid = std::min(pairs, g_sms3);
  k_layer_tail3<<<grid, kThreads, SMEM, st>>>(mp, a);
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

}  // namespace predtop
