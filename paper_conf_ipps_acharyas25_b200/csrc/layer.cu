// layer.cu -- K7: the post-attention half of the DAG-Transformer layer
// (Fig. 4; reading R6, post-LN encoder layer of [34]) as ONE
// persistent tcgen05 kernel per 128-row tile:
//     h  = LN1(x + att W_o^T + b_o)
//     x' = LN2(h + ReLU(h W_1^T + b_1) W_2^T + b_2)
// The d_ff-wide hidden activation never leaves the SM: it is produced in
// 128-column chunks into TMEM, turned into an fp16 UMMA operand in shared
// memory by the epilogue warps, and consumed by the FFN-2 MMAs that
// accumulate x' in TMEM.  HBM traffic per row: att (2d B) + x (4d B) in,
// x' (4d + 2d B) out.
//
// Roles (10 warps, one CTA per SM, persistent over row tiles):
//   warp 0      TMA producer: att tile, fp32 residual tile, and the weight
//               tiles (W_o, W_1 chunk, W_2 chunk; 64-wide K slices) through a
//               ring, in exactly the order the MMA warp consumes them
//   warp 1      MMA issuer (one thread): O-proj -> acc_o; FFN-1 chunk j ->
//               acc_f[j%2] (double buffered, so chunk j+1 overlaps the ReLU
//               epilogue of chunk j); FFN-2 chunk j -> acc_out (accumulated)
//   warps 2..9  epilogue: LN1 (acc_o + b_o + x -> h fp32 in place, h fp16 as
//               the FFN-1 A operand), ReLU(acc_f + b_1) -> fp16 A operand of
//               FFN-2, LN2 (acc_out + b_2 + h) -> x' fp32 / fp16, TMA stores
// TMEM columns: acc_o [0,D) | acc_f0 [D,D+128) | acc_f1 [D+128,D+256) |
//               acc_out [D+256, 2D+256)   (512 at D = 128)
#include <algorithm>

#include "internal.h"
#include "sm100.cuh"

namespace predtop {

#ifdef PREDTOP_TRACE
// Debug timeline of CTA 0 (first 16 tiles): %globaltimer at phase boundaries.
__device__ unsigned long long g_tail_trace[16][16];
__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define TTRACE(i, k) \
  do {               \
    if (leader && blockIdx.x == 0 && (i) < 16) g_tail_trace[i][k] = gtime(); \
  } while (0)
// per-warp clock64 at 4 points of FFN chunk 1 of tile 4 (CTA 0)
__device__ long long g_tail_trace2[4][16];
// MMA warp, tiles 2..9 of CTA 0: total clocks spent waiting on [0] ring_full,
// [1] p_ready, [2] h_ready, [3] a_full, [4] o_empty / out_empty; [5] tile span
__device__ long long g_tail_trace3[8];
#define TWAIT(k, stmt)                                                   \
  do {                                                                   \
    const long long t0_ = clock64();                                     \
    stmt;                                                                \
    if (blockIdx.x == 0 && tile_i >= 2 && tile_i < 10) g_tail_trace3[k] += clock64() - t0_; \
  } while (0)
#define TTRACEW(i, j, k) \
  do {                   \
    if (lane == 0 && blockIdx.x == 0 && (i) == 4 && (j) == 1) g_tail_trace2[k][warp - 2] = clock64(); \
  } while (0)
#else
#define TTRACEW(i, j, k) \
  do {                   \
  } while (0)
#define TWAIT(k, stmt) stmt
#define TTRACE(i, k) \
  do {               \
  } while (0)
#endif

namespace {

#ifndef PREDTOP_TAIL_GROUPS
#define PREDTOP_TAIL_GROUPS 4
#endif
constexpr int kGroups = PREDTOP_TAIL_GROUPS;  // column groups of the epilogue (x 4 warps each)
constexpr int kEpi = 128 * kGroups;           // epilogue threads
constexpr int kThreads = 64 + kEpi;
constexpr int FC = 128;  // FFN chunk (hidden columns per chunk)
constexpr int kSub = 128 * 128;  // bytes of one [128 rows x 64 fp16] or [128 x 32 fp32] sub-tile

template <int D>
struct TailCfg {
  static constexpr int X32 = 128 * D * 4;   // residual / h / x' fp32 tile
  static constexpr int SA = 128 * D * 2;    // att tile [128 x D] (O-proj A operand)
  static constexpr int SH = 128 * D * 2;    // h fp16 (FFN-1 A operand) / x' fp16 staging
  static constexpr int SLOT = (D > FC ? D : FC) * 64 * 2;
  static constexpr int PARAMS = (6 * D + 1024) * 4;  // bo g1 be1 b2 g2 be2 [D], b1 [<= 1024]
  static constexpr int FIXED = X32 + SA + SH + PARAMS + 1024;
  static constexpr int RS_FIT = (224 * 1024 - FIXED) / SLOT;
  static constexpr int RS = RS_FIT > 6 ? 6 : RS_FIT;
  static constexpr int SMEM = FIXED + RS * SLOT;
  static constexpr uint32_t TMEM_COLS = 512;
  static_assert(RS >= 2, "smem budget");
};

struct TailMaps {
  CUtensorMap att, x32, x16, wo, w1, w2;
};

struct TailArgs {
  int M, dff;
  const float *bo, *g1, *be1, *b1, *b2, *g2, *be2;
  float eps;
};

template <int D>
__global__ void __launch_bounds__(kThreads, 1) k_layer_tail(const __grid_constant__ TailMaps mp, TailArgs args) {
  using C = TailCfg<D>;
  constexpr int RS = C::RS;
  constexpr int KD = D / 64;  // 64-wide K slices of d
  extern __shared__ unsigned char dsm[];
  unsigned char* base = sm100::align1024(dsm);
  unsigned char* sX = base;                 // fp32 [128 x D], D/32 sub-tiles
  unsigned char* sA = sX + C::X32;          // att
  unsigned char* sH = sA + C::SA;           // h fp16 / x' fp16
  unsigned char* ring = sH + C::SH;
  float* sPar = reinterpret_cast<float*>(ring + RS * C::SLOT);  // per-layer vectors
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
  __shared__ __align__(8) uint64_t a_full, a_free, x_full, x_free, o_full, o_empty, h_ready;
  __shared__ __align__(8) uint64_t f_full[2], p_ready[2], out_full, out_empty;
  __shared__ uint32_t tmem_slot;
  __shared__ float red_a[kGroups][128], red_b[kGroups][128];

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ntiles = (int)ceil_div(args.M, 128);
  const int NJ = args.dff / FC;

  if (threadIdx.x == 0) {
    for (int s = 0; s < RS; ++s) {
      sm100::mbar_init(&ring_full[s], 1);
      sm100::mbar_init(&ring_empty[s], 1);
    }
    uint64_t* singles[] = {&a_full, &a_free, &x_full, &x_free, &o_full, &o_empty, &h_ready,
                           &f_full[0], &f_full[1], &p_ready[0], &p_ready[1],
                           &out_full, &out_empty};
    for (uint64_t* b : singles) sm100::mbar_init(b, 1);
    sm100::fence_mbar_init();
  }
  if (warp == 1) sm100::tmem_alloc<C::TMEM_COLS>(&tmem_slot);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem = tmem_slot;
  const uint32_t acc_o = tmem, acc_out = tmem + D + 2 * FC;

  if (warp == 0) {
    if (lane == 0) {  // ------------------------------------------ TMA producer
      sm100::tma_prefetch(&mp.att);
      sm100::tma_prefetch(&mp.x32);
      sm100::tma_prefetch(&mp.wo);
      sm100::tma_prefetch(&mp.w1);
      sm100::tma_prefetch(&mp.w2);
      int it = 0;
      auto load_w = [&](const CUtensorMap* m, int c0, int c1, int rows) {
        const int s = it % RS;
        sm100::mbar_wait(&ring_empty[s], ((it / RS) & 1) ^ 1);
        sm100::mbar_arrive_expect_tx(&ring_full[s], rows * 128);
        sm100::tma_load_2d(ring + s * C::SLOT, m, &ring_full[s], c0, c1);
        ++it;
      };
      int i = 0;
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
        const int m0 = t * 128;
        sm100::mbar_wait(&a_free, (i & 1) ^ 1);
        sm100::mbar_arrive_expect_tx(&a_full, 128 * D * 2);
        for (int b = 0; b < KD; ++b) sm100::tma_load_2d(sA + b * kSub, &mp.att, &a_full, b * 64, m0);
        for (int kc = 0; kc < KD; ++kc) load_w(&mp.wo, kc * 64, 0, D);
        sm100::mbar_wait(&x_free, i & 1);
        sm100::mbar_arrive_expect_tx(&x_full, 128 * D * 4);
        for (int b = 0; b < D / 32; ++b) sm100::tma_load_2d(sX + b * kSub, &mp.x32, &x_full, b * 32, m0);
        for (int j = 0; j < 2 && j < NJ; ++j)
          for (int kc = 0; kc < KD; ++kc) load_w(&mp.w1, kc * 64, j * FC, FC);
        for (int j = 0; j < NJ; ++j) {
          for (int kc = 0; kc < FC / 64; ++kc) load_w(&mp.w2, j * FC + kc * 64, 0, D);
          if (j + 2 < NJ)
            for (int kc = 0; kc < KD; ++kc) load_w(&mp.w1, kc * 64, (j + 2) * FC, FC);
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {  // ------------------------------------------ MMA issuer
      constexpr uint32_t id_D = sm100::make_idesc_f16(128, D);
      constexpr uint32_t id_F = sm100::make_idesc_f16(128, FC);
      int it = 0;
      int tile_i = 0;
      (void)tile_i;
      // consume `nk` ring slots: D[tmem] (+)= A (64-wide K slices at a_base + kc*kSub) * slot^T
      auto mma_ring = [&](uint32_t d_tmem, uint32_t a_base, int nk, uint32_t idesc, bool first) {
        for (int kc = 0; kc < nk; ++kc, ++it) {
          const int s = it % RS;
          TWAIT(0, sm100::mbar_wait(&ring_full[s], (it / RS) & 1));
          sm100::tc_fence_after();
          const uint32_t b0 = sm100::smem_u32(ring + s * C::SLOT);
          const uint32_t a0 = a_base + kc * kSub;
#pragma unroll
          for (int kk = 0; kk < 4; ++kk)
            sm100::mma_f16_ss(d_tmem, sm100::make_sdesc<128>(a0 + kk * 32),
                              sm100::make_sdesc<128>(b0 + kk * 32), idesc, !(first && kc == 0 && kk == 0));
          sm100::mma_commit(&ring_empty[s]);
        }
      };
      // FFN-2 with A = P from TMEM: the epilogue leaves ReLU(chunk) as fp16
      // pairs in the first FG/2 columns of each group's FG-column slice of
      // acc_f[b]; K-step ks (16 hidden units) sits at column pcol(ks).
      constexpr int FG = FC / kGroups;
      auto mma_ring_ts = [&](uint32_t d_tmem, uint32_t p_tmem, int nk, uint32_t idesc, bool first) {
        for (int kc = 0; kc < nk; ++kc, ++it) {
          const int s = it % RS;
          TWAIT(0, sm100::mbar_wait(&ring_full[s], (it / RS) & 1));
          sm100::tc_fence_after();
          const uint32_t b0 = sm100::smem_u32(ring + s * C::SLOT);
#pragma unroll
          for (int kk = 0; kk < 4; ++kk) {
            const int ks = 4 * kc + kk;
            const uint32_t pcol = (uint32_t)((ks / (FG / 16)) * FG + (ks % (FG / 16)) * 8);
            sm100::mma_f16_ts(d_tmem, p_tmem + pcol, sm100::make_sdesc<128>(b0 + kk * 32), idesc,
                              !(first && kc == 0 && kk == 0));
          }
          sm100::mma_commit(&ring_empty[s]);
        }
      };
      const uint32_t aA = sm100::smem_u32(sA), aH = sm100::smem_u32(sH);
      int i = 0;
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
        const int cbase = i * NJ;  // global FFN chunk counter of this tile's chunk 0
        // FFN-1 of chunk j into acc_f[j&1].  It overwrites the P of chunk j-2,
        // which FFN-2 of chunk j-2 reads from TMEM; that MMA was issued earlier
        // by this thread, and tcgen05.mma executes in issue order.
        auto ffn1 = [&](int j) {
          mma_ring(tmem + D + (j & 1) * FC, aH, KD, id_F, true);
          sm100::mma_commit(&f_full[j & 1]);
        };
        tile_i = i;
#ifdef PREDTOP_TRACE
        const long long tspan0 = clock64();
#endif
        TWAIT(3, sm100::mbar_wait(&a_full, i & 1));
        TWAIT(4, sm100::mbar_wait(&o_empty, (i & 1) ^ 1));
        sm100::tc_fence_after();
        mma_ring(acc_o, aA, KD, id_D, true);  // O-proj
        sm100::mma_commit(&o_full);
        sm100::mma_commit(&a_free);  // sA read: the next att tile may land
        TWAIT(2, sm100::mbar_wait(&h_ready, i & 1));
        sm100::tc_fence_after();
        for (int j = 0; j < 2 && j < NJ; ++j) ffn1(j);
        for (int j = 0; j < NJ; ++j) {
          const int b = j & 1, u = (cbase + j) >> 1;
          TWAIT(1, sm100::mbar_wait(&p_ready[b], u & 1));
          if (j == 0) TWAIT(4, sm100::mbar_wait(&out_empty, (i & 1) ^ 1));
          sm100::tc_fence_after();
          mma_ring_ts(acc_out, tmem + D + b * FC, FC / 64, id_D, j == 0);  // FFN-2 chunk j
          if (j + 2 < NJ) ffn1(j + 2);
        }
        sm100::mma_commit(&out_full);
#ifdef PREDTOP_TRACE
        if (blockIdx.x == 0 && i >= 2 && i < 10) g_tail_trace3[5] += clock64() - tspan0;
#endif
      }
    }
  } else {
    // ------------------------------------------ epilogue warps 2..(1 + 4 kGroups)
    const int q = warp & 3, grp = (warp - 2) >> 2;
    const int r = q * 32 + lane;
    const uint32_t lrow = (uint32_t)(q * 32) << 16;
    const bool leader = (warp == 2 && lane == 0);
    constexpr int DG = D / kGroups;  // columns of the row handled by this thread
    constexpr int FG = FC / kGroups;  // hidden columns of an FFN chunk per thread
    // One LayerNorm block of row r, this thread doing columns [grp*DG, +DG),
    // register resident: z = acc (TMEM) + bias + sX (fp32 residual), mean and
    // variance over the column groups through red_a / red_b, then
    // y = (z - mean) * rstd * g + be  ->  sX (fp32, in place) and sH (fp16).
    auto ln_block = [&](uint32_t acc, const float* bias, const float* g, const float* be) {
      float z[DG];
      sm100::tmem_ld<DG>(acc + lrow + grp * DG, z);
      sm100::tc_fence_before();
      float sum = 0.f;
#pragma unroll
      for (int k = 0; k < DG / 4; ++k) {
        const int c4 = grp * DG / 4 + k;
        const float4 x = *reinterpret_cast<const float4*>(sX + (c4 / 8) * kSub + sm100::swz<128>(r, c4 % 8));
        const float4 bb = reinterpret_cast<const float4*>(bias)[c4];
        z[4 * k + 0] = x.x + (z[4 * k + 0] + bb.x);
        z[4 * k + 1] = x.y + (z[4 * k + 1] + bb.y);
        z[4 * k + 2] = x.z + (z[4 * k + 2] + bb.z);
        z[4 * k + 3] = x.w + (z[4 * k + 3] + bb.w);
        sum += (z[4 * k] + z[4 * k + 1]) + (z[4 * k + 2] + z[4 * k + 3]);
      }
      red_a[grp][r] = sum;
      sm100::named_bar<kEpi>(1);
      float tot = 0.f;
#pragma unroll
      for (int i2 = 0; i2 < kGroups; ++i2) tot += red_a[i2][r];
      const float mean = tot * (1.0f / D);
      float sq = 0.f;
#pragma unroll
      for (int k = 0; k < DG / 4; ++k) {
        const float a = z[4 * k] - mean, b = z[4 * k + 1] - mean, cc = z[4 * k + 2] - mean, d = z[4 * k + 3] - mean;
        sq += (a * a + b * b) + (cc * cc + d * d);
      }
      red_b[grp][r] = sq;
      sm100::named_bar<kEpi>(1);
      float tsq = 0.f;
#pragma unroll
      for (int i2 = 0; i2 < kGroups; ++i2) tsq += red_b[i2][r];
      const float rstd = rsqrtf(tsq * (1.0f / D) + args.eps);
#pragma unroll
      for (int k8 = 0; k8 < DG / 8; ++k8) {
        float y[8];
#pragma unroll
        for (int h2 = 0; h2 < 2; ++h2) {
          const int k = 2 * k8 + h2, c4 = grp * DG / 4 + k;
          const float4 gm = reinterpret_cast<const float4*>(g)[c4];
          const float4 bt = reinterpret_cast<const float4*>(be)[c4];
          float4 o;
          o.x = (z[4 * k + 0] - mean) * rstd * gm.x + bt.x;
          o.y = (z[4 * k + 1] - mean) * rstd * gm.y + bt.y;
          o.z = (z[4 * k + 2] - mean) * rstd * gm.z + bt.z;
          o.w = (z[4 * k + 3] - mean) * rstd * gm.w + bt.w;
          *reinterpret_cast<float4*>(sX + (c4 / 8) * kSub + sm100::swz<128>(r, c4 % 8)) = o;
          y[4 * h2] = o.x; y[4 * h2 + 1] = o.y; y[4 * h2 + 2] = o.z; y[4 * h2 + 3] = o.w;
        }
        const int c = grp * DG + 8 * k8;
        *reinterpret_cast<uint4*>(sH + (c / 64) * kSub + sm100::swz<128>(r, (c % 64) / 8)) =
            make_uint4(sm100::pack_half2(y[0], y[1]), sm100::pack_half2(y[2], y[3]),
                       sm100::pack_half2(y[4], y[5]), sm100::pack_half2(y[6], y[7]));
      }
    };
    int i = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
      const int m0 = t * 128;
      const int cbase = i * NJ;
      // previous tile's stores have read sX / sH -> the residual of this tile may land
      TTRACE(i, 0);
      if (leader) sm100::bulk_wait_read0();
      sm100::named_bar<kEpi>(1);
      if (leader) sm100::mbar_arrive(&x_free);
      TTRACE(i, 1);
      // ---- LN1
      sm100::mbar_wait(&o_full, i & 1);
      TTRACE(i, 2);
      sm100::mbar_wait(&x_full, i & 1);
      TTRACE(i, 3);
      sm100::tc_fence_after();
      ln_block(acc_o, p_bo, p_g1, p_be1);
      sm100::fence_proxy_async();
      sm100::named_bar<kEpi>(1);
      if (leader) {
        sm100::mbar_arrive(&o_empty);
        sm100::mbar_arrive(&h_ready);
      }
      TTRACE(i, 4);
      // ---- FFN chunks: ReLU(acc_f + b_1) -> fp16 pairs back into acc_f (the
      // first half of this thread's column slice): the TMEM A operand of FFN-2
      for (int j = 0; j < NJ; ++j) {
        const int b = j & 1, u = (cbase + j) >> 1;
        sm100::mbar_wait(&f_full[b], u & 1);
        TTRACE(i, 5 + 2 * (j & 3));
        TTRACEW(i, j, 0);
        sm100::tc_fence_after();
        const uint32_t accf = tmem + D + b * FC + lrow + grp * FG;
        const float* b1 = p_b1 + j * FC + grp * FG;
        float v[FG];
        sm100::tmem_ld<FG>(accf, v);
        TTRACEW(i, j, 1);
        uint32_t pk[FG / 2];
#pragma unroll
        for (int k = 0; k < FG / 4; ++k) {
          const float4 bb = reinterpret_cast<const float4*>(b1)[k];
          pk[2 * k] = sm100::pack_half2(fmaxf(v[4 * k] + bb.x, 0.f), fmaxf(v[4 * k + 1] + bb.y, 0.f));
          pk[2 * k + 1] = sm100::pack_half2(fmaxf(v[4 * k + 2] + bb.z, 0.f), fmaxf(v[4 * k + 3] + bb.w, 0.f));
        }
#pragma unroll
        for (int k = 0; k < FG / 32; ++k) sm100::tmem_st16(accf + 16 * k, pk + 16 * k);
        sm100::tmem_wait_st();
        TTRACEW(i, j, 2);
        sm100::tc_fence_before();
        TTRACEW(i, j, 3);
        sm100::named_bar<kEpi>(1);
        if (leader) sm100::mbar_arrive(&p_ready[b]);
        TTRACE(i, 6 + 2 * (j & 3));
      }
      // ---- LN2 and stores
      sm100::mbar_wait(&out_full, i & 1);
      TTRACE(i, 13);
      sm100::tc_fence_after();
      ln_block(acc_out, p_b2, p_g2, p_be2);
      sm100::fence_proxy_async();
      sm100::named_bar<kEpi>(1);
      if (leader) {
        sm100::mbar_arrive(&out_empty);
        for (int b = 0; b < D / 32; ++b) sm100::tma_store_2d(&mp.x32, sX + b * kSub, b * 32, m0);
        for (int b = 0; b < KD; ++b) sm100::tma_store_2d(&mp.x16, sH + b * kSub, b * 64, m0);
        sm100::bulk_commit();
      }
      TTRACE(i, 14);
    }
    if (leader) sm100::bulk_wait0();
  }
  __syncwarp();
  sm100::tc_fence_before();
  __syncthreads();
  if (warp == 1) sm100::tmem_dealloc<C::TMEM_COLS>(tmem);
}


template <int D>
predtop_status launch_d(const TailMaps& mp, const TailArgs& a, cudaStream_t st) {
  using C = TailCfg<D>;
  PT_SMEM_ATTR(k_layer_tail<D>, C::SMEM);
  const int g_sms = num_sms();
  if (!g_sms) return PREDTOP_ERR_CUDA;
  const int grid = (int)std::min<int64_t>(ceil_div(a.M, 128), g_sms);
  k_layer_tail<D><<<grid, kThreads, C::SMEM, st>>>(mp, a);
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

}  // namespace

bool layer_tail_supported(int d, int dff) { return (d == 64 || d == 128) && dff % (2 * FC) == 0; }

predtop_status layer_tail_launch(const predtop_model_s* m, int l, const __half* att, float* x32,
                                 __half* x16, int M, cudaStream_t st) {
  const int d = m->cfg.d_model, dff = m->cfg.d_ff;
  if (!layer_tail_supported(d, dff)) {
    set_error("fused layer tail needs d in {64,128} and d_ff %% 256 == 0");
    return PREDTOP_ERR_UNSUPPORTED;
  }
  if (M <= 0) return PREDTOP_OK;
  const LayerDev& L = m->layer[l];
  TailMaps mp;
  if (!encode_tma_2d(&mp.att, att, 2, d, M, 64, 128) || !encode_tma_2d(&mp.x32, x32, 4, d, M, 32, 128) ||
      !encode_tma_2d(&mp.x16, x16, 2, d, M, 64, 128))
    return PREDTOP_ERR_CUDA;
  mp.wo = L.tm_o;
  mp.w1 = L.tm_1c;
  mp.w2 = L.tm_2;
  TailArgs a{M, dff, L.bo, L.g1, L.be1, L.b1, L.b2, L.g2, L.be2, m->cfg.ln_eps};
  return d == 128 ? launch_d<128>(mp, a, st) : launch_d<64>(mp, a, st);
}

}  // namespace predtop

#ifdef PREDTOP_TRACE
extern "C" PREDTOP_API int predtop_debug_tail_trace(unsigned long long* out) {
  if (cudaMemcpyFromSymbol(out, predtop::g_tail_trace, sizeof(predtop::g_tail_trace)) != cudaSuccess) return -7;
  if (cudaMemcpyFromSymbol(out + 256, predtop::g_tail_trace2, sizeof(predtop::g_tail_trace2)) != cudaSuccess) return -7;
  return cudaMemcpyFromSymbol(out + 320, predtop::g_tail_trace3, sizeof(predtop::g_tail_trace3)) == cudaSuccess ? 0 : -7;
}
#endif
