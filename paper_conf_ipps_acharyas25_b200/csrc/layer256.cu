// layer256.cu -- K7 at d = 256 (the MoE config): the post-attention half of
// the DAG-Transformer layer (Fig. 4; reading R6, post-LN encoder
// layer of [34]),
//     h  = LN1(x + att W_o^T + b_o)
//     x' = LN2(h + ReLU(h W_1^T + b_1) W_2^T + b_2),
// as ONE persistent tcgen05 kernel per layer, so the d_ff-wide hidden
// activation never leaves the SM (the three-GEMM path wrote and re-read it
// through HBM: 2 x 1.6 GB per layer on the MoE batch).
//
// One CTA per SM (all 512 TMEM columns), one 128-row tile at a time:
//   TMEM  acc [0, 256): the O-projection; after LN1 the epilogue writes
//         h + b_2 back into it (tcgen05.st) so FFN-2 accumulates onto the
//         residual: acc = h + b_2 + FFN(h), the LN2 input.
//         acc_f[b] = [256 + 128 b, +128): FFN-1 chunk j (128 hidden units) in
//         buffer j & 1, turned in place into the fp16 ReLU output P_j that
//         FFN-2 reads as its A operand from tensor memory (TS-MMA).
//   SMEM  AH (64 KB, four SW128 K-slices): h (the FFN-1 A operand), and
//         after FFN-1 the per-warp staging of the x' TMA stores; a 4-unit
//         ring of 32 KB units (att halves and W_o K-slices, the fp32 residual
//         tile, W_1 / W_2 chunk halves, in consumption order).  Biases and LN
//         parameters are read from global memory (L1).
//   warp 0 TMA producer, warp 1 MMA issuer, warps 2..17 epilogue: lane quarter
//   q = warp % 4 -> rows 32q.., column group cg = (warp - 2) / 4 -> the 64
//   columns [64 cg, +64) of acc and the 32 hidden units [32 cg, +32) of an
//   FFN chunk.
// MMA per tile: O-proj 16 x (N=256, K=16), FFN-1 8 chunks x 16 x (N=128),
// FFN-2 8 x 8 x (N=256, A in TMEM) = 2.3 x 10^8 MACs... 151 MFLOP per tile.
#include <algorithm>

#include "internal.h"
#include "sm100.cuh"

namespace predtop {

#ifdef PREDTOP_TRACE
__device__ unsigned long long g_l256[16][16];  // CTA 0, tiles 0..15: clock64 at pipeline events
__device__ unsigned long long g_l256w[16][16][12];  // CTA 0, tiles 0..15, epilogue warps: LN events
__device__ __forceinline__ unsigned long long l256_clk() {  // memory clobber: stays between the loads/stores around it
  unsigned long long t;
  asm volatile("mov.u64 %0, %%clock64;" : "=l"(t)::"memory");
  return t;
}
#define LT(i, k)                                                 \
  do {                                                           \
    if (blockIdx.x == 0 && (i) < 16) g_l256[i][k] = l256_clk(); \
  } while (0)
#define LW(i, k)                                                                  \
  do {                                                                            \
    if (blockIdx.x == 0 && (i) < 16 && lane == 0) g_l256w[i][ew][k] = l256_clk(); \
  } while (0)
#else
#define LW(i, k) \
  do {           \
  } while (0)
#define LT(i, k) \
  do {           \
  } while (0)
#endif

#ifndef PREDTOP_L256_OUTW
#define PREDTOP_L256_OUTW 1  // x' leaves in 128-byte-row boxes (0: 16-column pieces)
#endif
#ifndef PREDTOP_L256_PF
#define PREDTOP_L256_PF 1  // L2 prefetch of the next tile's x and att during this tile's FFN (0: off)
#endif
#ifndef PREDTOP_L256_STG
#define PREDTOP_L256_STG 0  // 1: x' leaves through coalesced STG instead of TMA stores (A/B)
#endif

namespace {

constexpr int D = 256;
constexpr int FC = 128;               // FFN chunk (hidden units), two TMEM buffers
constexpr int RS = 4;                 // ring units
constexpr int UNIT = 32 * 1024;       // bytes of one ring unit
constexpr int KSL = 128 * 128;        // one [128 rows x 64 fp16] SW128 K-slice (16 KB)
constexpr int AHB = 4 * KSL;          // att / h tile
constexpr int kEpiWarps = 16;
constexpr int kEpi = 32 * kEpiWarps;
constexpr int kThreads = 64 + kEpi;
constexpr int kMaxFF = 4096;
constexpr int STG32 = 32 * 16 * 4;    // per-warp x' staging in AH: [32 rows x 16 fp32] (SW64)
constexpr int STG16 = 32 * 16 * 2;    //                           [32 rows x 16 fp16] (SW32)
static_assert(kEpiWarps * (STG32 + STG16) <= AHB, "x' staging lives in the h tile");
constexpr int STGW = 32 * 128;       // PREDTOP_L256_OUTW: one [32 rows x 128 B] SW128 box per warp
static_assert(kEpiWarps * STGW <= AHB, "x' staging lives in the h tile");
constexpr int SMEM = 1024 + RS * UNIT + AHB;
static_assert(SMEM <= 227 * 1024, "one CTA per SM");

struct T256Maps {
  CUtensorMap att, x32in, wo, w1, w2, x32out, x16out;
};

struct T256Args {
  int M, dff;
  const float *bo, *g1, *be1, *b1, *b2, *g2, *be2;
  float eps;
  float* x32;   // residual stream [M][D] fp32 (read through x32in, then overwritten with x')
  __half* x16;  // its fp16 shadow [M][D]
};

__global__ void __launch_bounds__(kThreads, 1) k_layer_tail256(const __grid_constant__ T256Maps mp, T256Args args) {
  extern __shared__ unsigned char dsm[];
  unsigned char* base = sm100::align1024(dsm);
  unsigned char* ring = base;               // RS x 32 KB
  unsigned char* sAH = ring + RS * UNIT;    // [4 K-slices][128 rows x 64] fp16, SW128
  unsigned char* sStg = sAH;                // x' staging (per epilogue warp STG32 + STG16), once h is dead
  // the D-length biases and LN parameters in shared memory (broadcast
  // reads; through L1 they are evicted by the epilogue's spill traffic and
  // every LayerNorm piece waits on L2); b_1 (d_ff long, read once per FFN
  // chunk) stays in global memory
  __shared__ __align__(16) float sPar[6][D];
  const float* p_bo = sPar[0];
  const float* p_g1 = sPar[1];
  const float* p_be1 = sPar[2];
  const float* p_b2 = sPar[3];
  const float* p_g2 = sPar[4];
  const float* p_be2 = sPar[5];
  const float* __restrict__ p_b1 = args.b1;
  __shared__ __align__(8) uint64_t ring_full[RS], ring_empty[RS];
  __shared__ __align__(8) uint64_t o_full, o_empty, h_ready, out_full;
  __shared__ __align__(8) uint64_t f_full[2], p_ready[2];  // per acc_f buffer
  __shared__ uint32_t tmem_slot;
  __shared__ float red[2][4][128];   // LN1 row statistics
  __shared__ float red2[2][4][128];  // LN2 row statistics (LN1 of the next tile may overlap their reads)

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ntiles = (int)ceil_div(args.M, 128);
  const int NJ = args.dff / FC;
  // ring units per tile: att 2 + W_o 4 (order att_a Wo0 Wo1 att_b Wo2 Wo3),
  // x 4, W_1 2 per chunk, W_2 2 per chunk
  const int UPT = 10 + 4 * NJ;

  if (threadIdx.x == 0) {
    for (int s = 0; s < RS; ++s) {
      sm100::mbar_init(&ring_full[s], 1);
      sm100::mbar_init(&ring_empty[s], 1);
    }
    uint64_t* singles[] = {&o_full, &o_empty, &h_ready, &out_full, &f_full[0], &f_full[1]};
    for (uint64_t* b : singles) sm100::mbar_init(b, 1);
    sm100::mbar_init(&p_ready[0], kEpiWarps);  // one arrival per epilogue warp
    sm100::mbar_init(&p_ready[1], kEpiWarps);
    sm100::fence_mbar_init();
  }
  if (warp == 1) sm100::tmem_alloc<512>(&tmem_slot);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem = tmem_slot;
  const uint32_t acc = tmem, acc_f = tmem + D;

  if (warp == 0) {
    if (lane == 0) {  // ------------------------------------------ TMA producer
      sm100::tma_prefetch(&mp.att);
      sm100::tma_prefetch(&mp.x32in);
      sm100::tma_prefetch(&mp.wo);
      sm100::tma_prefetch(&mp.w1);
      sm100::tma_prefetch(&mp.w2);
      int it = 0;
      auto unit = [&]() -> unsigned char* {  // claim the next ring unit (expects UNIT bytes)
        const int s = it % RS;
        sm100::mbar_wait(&ring_empty[s], ((it / RS) & 1) ^ 1);
        sm100::mbar_arrive_expect_tx(&ring_full[s], UNIT);
        return ring + s * UNIT;
      };
      int i = 0;
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
        const int m0 = t * 128;
        // att half a (K-slices 2a, 2a+1: two [128 x 64] boxes), then the two
        // W_o K-slices [256 out x 64 in] it multiplies
        for (int a = 0; a < 2; ++a) {
          unsigned char* u = unit();
          for (int sub = 0; sub < 2; ++sub)
            sm100::tma_load_2d(u + sub * KSL, &mp.att, &ring_full[it % RS], 64 * (2 * a + sub), m0);
          ++it;
          for (int sub = 0; sub < 2; ++sub) {
            unsigned char* w = unit();
            sm100::tma_load_2d(w, &mp.wo, &ring_full[it % RS], 64 * (2 * a + sub), 0);
            ++it;
          }
        }
        // the residual x: unit cg = columns [64cg, +64) as two [128 x 32] fp32 boxes
        for (int cg = 0; cg < 4; ++cg) {
          unsigned char* u = unit();
          sm100::tma_load_2d(u, &mp.x32in, &ring_full[it % RS], 64 * cg, m0);
          sm100::tma_load_2d(u + KSL, &mp.x32in, &ring_full[it % RS], 64 * cg + 32, m0);
          ++it;
        }
        // FFN weights in MMA order: F1_0 F1_1 F2_0 F1_2 F2_1 ... F2_{NJ-1}.
        // W_1 chunk j half a: rows [128j, +128) x K-slices {2a, 2a+1};
        // W_2 chunk j half a: rows [0, 256) x K-slice (2j + a) of the hidden dim
        auto load_w1 = [&](int j) {
          for (int a = 0; a < 2; ++a) {
            unsigned char* u = unit();
            for (int sub = 0; sub < 2; ++sub)
              sm100::tma_load_2d(u + sub * KSL, &mp.w1, &ring_full[it % RS], 64 * (2 * a + sub), FC * j);
            ++it;
          }
        };
        auto load_w2 = [&](int j) {
          for (int a = 0; a < 2; ++a) {
            unsigned char* u = unit();
            sm100::tma_load_2d(u, &mp.w2, &ring_full[it % RS], FC * j + 64 * a, 0);
            ++it;
          }
        };
        // PREDTOP_L256_PF: the next tile's residual x (8 boxes, 128 KB fp32)
        // and att (4 boxes, 64 KB) prefetched into L2, spread over this
        // tile's FFN chunks behind their weight loads: the ring frees their
        // units only after the O-projection, and from HBM at one SM's share of
        // the bandwidth the x tile alone cost ~5k cycles of LN1 wait
        const bool pf = PREDTOP_L256_PF && t + (int)gridDim.x < ntiles;
        const int m1 = (t + (int)gridDim.x) * 128;
        int pfb = 0;
        auto prefetch_upto = [&](int nb) {
          for (; pfb < nb; ++pfb) {
            if (pfb < D / 32) sm100::tma_prefetch_l2_2d(&mp.x32in, 32 * pfb, m1);
            else sm100::tma_prefetch_l2_2d(&mp.att, 64 * (pfb - D / 32), m1);
          }
        };
        load_w1(0);
        for (int j = 0; j < NJ; ++j) {
          if (j + 1 < NJ) load_w1(j + 1);
          load_w2(j);
          if (pf) prefetch_upto(((j + 1) * (D / 32 + 4)) / NJ);
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {  // ------------------------------------------ MMA issuer
      constexpr uint32_t id_N256 = sm100::make_idesc_f16(128, 256);
      constexpr uint32_t id_N128 = sm100::make_idesc_f16(128, FC);
      const uint32_t aAH = sm100::smem_u32(sAH), aRing = sm100::smem_u32(ring);
      int it = 0, i = 0;
      auto unit_wait = [&]() -> uint32_t {
        const int s = it % RS;
        sm100::mbar_wait(&ring_full[s], (it / RS) & 1);
        sm100::tc_fence_after();
        return aRing + s * UNIT;
      };
      auto unit_free = [&]() {
        sm100::mma_commit(&ring_empty[it % RS]);
        ++it;
      };
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
        // ---- O-projection: acc = att W_o^T (acc free once LN2 of the previous tile read it)
        LT(i, 0);
        sm100::mbar_wait(&o_empty, (i & 1) ^ 1);
        LT(i, 1);
        sm100::tc_fence_after();
        for (int a = 0; a < 2; ++a) {
          const int ia = it;  // the att unit stays until both W_o units of this half are consumed
          const uint32_t a0 = unit_wait();
          ++it;
          for (int sub = 0; sub < 2; ++sub) {
            const uint32_t b0 = unit_wait();
#pragma unroll
            for (int kk = 0; kk < 4; ++kk)
              sm100::mma_f16_ss(acc, sm100::make_sdesc<128>(a0 + sub * KSL + kk * 32),
                                sm100::make_sdesc<128>(b0 + kk * 32), id_N256, (a | sub | kk) != 0);
            unit_free();
          }
          sm100::mma_commit(&ring_empty[ia % RS]);
        }
        sm100::mma_commit(&o_full);
        LT(i, 2);
        // the 4 x units belong to the epilogue (it frees them after LN1).
        // Skipping them here is safe: the next unit_wait (FFN-1, after
        // h_ready) is on a phase whose predecessor the epilogue consumed
        it += 4;
        // ---- FFN: acc holds h + b_2, AH holds h (written by the epilogue after LN1)
        sm100::mbar_wait(&h_ready, i & 1);
        LT(i, 3);
        sm100::tc_fence_after();
        auto ffn1 = [&](int j) {
          const uint32_t dst = acc_f + (uint32_t)((j & 1) * FC);
          for (int a = 0; a < 2; ++a) {
            const uint32_t b0 = unit_wait();
#pragma unroll
            for (int sub = 0; sub < 2; ++sub)
#pragma unroll
              for (int kk = 0; kk < 4; ++kk)
                sm100::mma_f16_ss(dst, sm100::make_sdesc<128>(aAH + (2 * a + sub) * KSL + kk * 32),
                                  sm100::make_sdesc<128>(b0 + sub * KSL + kk * 32), id_N128, (a | sub | kk) != 0);
            unit_free();
          }
          sm100::mma_commit(&f_full[j & 1]);
        };
        ffn1(0);
        for (int j = 0; j < NJ; ++j) {
          if (j + 1 < NJ) ffn1(j + 1);  // keeps the tensor pipe busy during ReLU_j
          // FFN-2 chunk j: acc += P_j W_2[:, chunk]^T, P_j from TMEM.  Epilogue
          // group cg leaves hidden units [32cg, +32) as 16 packed fp16 columns
          // at 32cg of the buffer: K-step ks sits at 32(ks/2) + 8(ks%2).
          sm100::mbar_wait(&p_ready[j & 1], ((i * NJ + j) >> 1) & 1);
          sm100::tc_fence_after();
          const uint32_t src = acc_f + (uint32_t)((j & 1) * FC);
          for (int a = 0; a < 2; ++a) {
            const uint32_t b0 = unit_wait();
#pragma unroll
            for (int kk = 0; kk < 4; ++kk) {
              const int ks = 4 * a + kk;
              sm100::mma_f16_ts(acc, src + (uint32_t)(32 * (ks / 2) + 8 * (ks % 2)),
                                sm100::make_sdesc<128>(b0 + kk * 32), id_N256, 1u);
            }
            unit_free();
          }
        }
        sm100::mma_commit(&out_full);
        LT(i, 4);
      }
    }
  } else {
    // ------------------------------------------ epilogue warps 2..17
    const int ew = warp - 2;
    const int q = warp & 3, cg = ew >> 2;
    const int r = q * 32 + lane;  // tile row of this thread (TMEM lane)
    const uint32_t lrow = (uint32_t)(q * 32) << 16;
    const bool leader = (ew == 0 && lane == 0);
    {
      const float* src[6] = {args.bo, args.g1, args.be1, args.b2, args.g2, args.be2};
#pragma unroll
      for (int k = 0; k < 6; ++k)
        if (ew * 32 + lane < D) sPar[k][ew * 32 + lane] = src[k][ew * 32 + lane];
      sm100::named_bar<kEpi>(1);
    }
    int i = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
      const int m0 = t * 128;
      const int cbase = i * NJ;
      // ---- LN1: z = x + acc + b_o, two passes over 16-column pieces (the
      // residual x stays in its ring unit, acc in TMEM: no 64-value register
      // array, which would not fit the 96 registers of an 18-warp CTA).
      // o_full first: the O-projection consumed this tile's W_o units, i.e.
      // the previous phase of each x unit completed, so the parity wait is
      // never two phases ahead (it would alias and return at once)
      sm100::mbar_wait(&o_full, i & 1);
      if (leader) LT(i, 5); LW(i, 0);
      const int xit = i * UPT + 6;
      const int itk = xit + cg;
      sm100::mbar_wait(&ring_full[itk % RS], (itk / RS) & 1);
      if (leader) LT(i, 6); LW(i, 1);
      sm100::tc_fence_after();
      const unsigned char* xu = ring + (itk % RS) * UNIT;  // columns [64cg, +64): two [128 x 32] fp32 boxes
      // z = acc + x + b_o for this thread's 64 columns, kept in registers
      // across the statistics barrier (one TMEM read: all four loads in
      // flight, one wait)
      float z[64];
      sm100::tmem_ld<64>(acc + lrow + 64 * cg, z);
#pragma unroll
      for (int k = 0; k < 2; ++k)
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          const float4 v = *reinterpret_cast<const float4*>(xu + k * KSL + sm100::swz<128>(r, c));
          const float4 bo = (*reinterpret_cast<const float4*>(p_bo + 64 * cg + 32 * k + 4 * c));
          float* zz = z + 32 * k + 4 * c;
          zz[0] += v.x + bo.x;
          zz[1] += v.y + bo.y;
          zz[2] += v.z + bo.z;
          zz[3] += v.w + bo.w;
        }
      float mean, rstd;
      {
        float s = 0.f, sq = 0.f;
#pragma unroll
        for (int e = 0; e < 64; ++e) {
          s += z[e];
          sq = fmaf(z[e], z[e], sq);
        }
        red[0][cg][r] = s;
        red[1][cg][r] = sq;
        if (leader) LT(i, 7); LW(i, 2);
        // h overwrites all of AH below: every warp's x' stores of the
        // previous tile (staged in AH) must have read it (before the barrier)
        if (lane == 0) sm100::bulk_wait_read0();
        __syncwarp();
        sm100::named_bar<kEpi>(1);
        if (leader) LT(i, 12); LW(i, 3);
        mean = ((red[0][0][r] + red[0][1][r]) + (red[0][2][r] + red[0][3][r])) * (1.0f / D);
        const float ex2 = ((red[1][0][r] + red[1][1][r]) + (red[1][2][r] + red[1][3][r])) * (1.0f / D);
        rstd = rsqrtf(fmaxf(ex2 - mean * mean, 0.f) + args.eps);
      }
      // h (fp16) -> AH K-slice cg (FFN-1 of the previous tile, the last
      // reader of its h, completed before that tile's out_full); h + b_2 ->
      // acc (FFN-2 accumulates onto it)
      unsigned char* hs = sAH + cg * KSL;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        float* zk = z + 16 * k;
        uint32_t hb[16], hp[8];
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          const int col = 64 * cg + 16 * k + 4 * c;
          const float4 g = (*reinterpret_cast<const float4*>(p_g1 + col));
          const float4 be = (*reinterpret_cast<const float4*>(p_be1 + col));
          const float4 b2 = (*reinterpret_cast<const float4*>(p_b2 + col));
          const float gg[4] = {g.x, g.y, g.z, g.w}, bb[4] = {be.x, be.y, be.z, be.w}, b22[4] = {b2.x, b2.y, b2.z, b2.w};
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            zk[4 * c + e] = (zk[4 * c + e] - mean) * rstd * gg[e] + bb[e];
            hb[4 * c + e] = __float_as_uint(zk[4 * c + e] + b22[e]);
          }
        }
#pragma unroll
        for (int e = 0; e < 8; ++e) hp[e] = sm100::pack_half2(zk[2 * e], zk[2 * e + 1]);
        *reinterpret_cast<uint4*>(hs + sm100::swz<128>(r, 2 * k)) = make_uint4(hp[0], hp[1], hp[2], hp[3]);
        *reinterpret_cast<uint4*>(hs + sm100::swz<128>(r, 2 * k + 1)) = make_uint4(hp[4], hp[5], hp[6], hp[7]);
        sm100::tmem_st16(acc + lrow + 64 * cg + 16 * k, hb);
      }
      if (leader) LT(i, 13); LW(i, 4);
      sm100::tmem_wait_st();
      sm100::fence_proxy_async();  // h writes (and the x reads) before the async proxy
      sm100::tc_fence_before();
      sm100::named_bar<kEpi>(1);
      if (leader) {
        for (int k = 0; k < 4; ++k) sm100::mbar_arrive(&ring_empty[(xit + k) % RS]);  // x units free
        sm100::mbar_arrive(&h_ready);
        LT(i, 8);
      }
      LW(i, 5);
      // ---- FFN chunks: ReLU(acc_f + b_1) -> fp16 pairs back into acc_f
      for (int j = 0; j < NJ; ++j) {
        const int cj = cbase + j;
        sm100::mbar_wait(&f_full[j & 1], (cj >> 1) & 1);
        sm100::tc_fence_after();
        {
          const uint32_t buf = acc_f + (uint32_t)((j & 1) * FC);
          float v[32];
          sm100::tmem_ld<32>(buf + lrow + 32 * cg, v);
          const float4* b1 = reinterpret_cast<const float4*>(p_b1 + j * FC + 32 * cg);
          uint32_t pk[16];
#pragma unroll
          for (int k = 0; k < 8; ++k) {
            const float4 b = __ldg(b1 + k);
            pk[2 * k] = sm100::pack_half2(fmaxf(v[4 * k] + b.x, 0.f), fmaxf(v[4 * k + 1] + b.y, 0.f));
            pk[2 * k + 1] = sm100::pack_half2(fmaxf(v[4 * k + 2] + b.z, 0.f), fmaxf(v[4 * k + 3] + b.w, 0.f));
          }
          sm100::tmem_st16(buf + lrow + 32 * cg, pk);
        }
        sm100::tmem_wait_st();
        sm100::tc_fence_before();
        __syncwarp();
        if (lane == 0) sm100::mbar_arrive(&p_ready[j & 1]);  // this warp's part of P_j is in TMEM
      }
      // ---- LN2: z = acc (= h + b_2 + FFN(h)), two passes over 16-column
      // pieces of TMEM; x' (fp32) and its fp16 shadow go straight from
      // registers to global memory (the stores drain during the next tile)
      if (leader) LT(i, 9);
      sm100::mbar_wait(&out_full, i & 1);
      if (leader) LT(i, 10); LW(i, 6);
      sm100::tc_fence_after();
      // the row's 64 values in registers (one TMEM read), so acc is free for
      // the next tile's O-projection as soon as every thread has read it
      sm100::tmem_ld<64>(acc + lrow + 64 * cg, z);
      sm100::tc_fence_before();
      {
        float s = 0.f, sq = 0.f;
#pragma unroll
        for (int e = 0; e < 64; ++e) {
          s += z[e];
          sq = fmaf(z[e], z[e], sq);
        }
        red2[0][cg][r] = s;
        red2[1][cg][r] = sq;
        sm100::named_bar<kEpi>(1);  // every epilogue thread has read acc (and written red) ...
        if (leader) LT(i, 14); LW(i, 8);
        if (leader) sm100::mbar_arrive(&o_empty);  // ... so the next O-projection may overwrite it
        mean = ((red2[0][0][r] + red2[0][1][r]) + (red2[0][2][r] + red2[0][3][r])) * (1.0f / D);
        const float ex2 = ((red2[1][0][r] + red2[1][1][r]) + (red2[1][2][r] + red2[1][3][r])) * (1.0f / D);
        rstd = rsqrtf(fmaxf(ex2 - mean * mean, 0.f) + args.eps);
      }
#if PREDTOP_L256_OUTW
      // pass B: normalise the 64 values in place, then three 128-byte-row
      // TMA boxes through this warp's 4 KB of AH (SW128: conflict-free
      // writes): x' columns [64cg, +32), [64cg + 32, +32) in fp32, then all
      // 64 columns in fp16.  Wide rows: the TMA store cost grows with the
      // number of box rows (16-column pieces took 2.7x as many)
#pragma unroll
      for (int c = 0; c < 16; ++c) {
        const int col = 64 * cg + 4 * c;
        const float4 g = (*reinterpret_cast<const float4*>(p_g2 + col));
        const float4 be = (*reinterpret_cast<const float4*>(p_be2 + col));
        z[4 * c] = (z[4 * c] - mean) * rstd * g.x + be.x;
        z[4 * c + 1] = (z[4 * c + 1] - mean) * rstd * g.y + be.y;
        z[4 * c + 2] = (z[4 * c + 2] - mean) * rstd * g.z + be.z;
        z[4 * c + 3] = (z[4 * c + 3] - mean) * rstd * g.w + be.w;
      }
      LW(i, 9);
      unsigned char* sw = sStg + ew * STGW;
#pragma unroll
      for (int p = 0; p < 3; ++p) {
        if (p == 2 && args.x16 == nullptr) break;  // last layer: no fp16 shadow
        if (p > 0) {
          if (lane == 0) sm100::bulk_wait_read0();
          __syncwarp();
          if (p == 1) LW(i, 10);
          if (p == 2) LW(i, 11);
        }
        if (p < 2) {
#pragma unroll
          for (int c = 0; c < 8; ++c)
            *reinterpret_cast<float4*>(sw + sm100::swz<128>(lane, c)) =
                make_float4(z[32 * p + 4 * c], z[32 * p + 4 * c + 1], z[32 * p + 4 * c + 2], z[32 * p + 4 * c + 3]);
        } else {
#pragma unroll
          for (int c = 0; c < 8; ++c)
            *reinterpret_cast<uint4*>(sw + sm100::swz<128>(lane, c)) =
                make_uint4(sm100::pack_half2(z[8 * c], z[8 * c + 1]), sm100::pack_half2(z[8 * c + 2], z[8 * c + 3]),
                           sm100::pack_half2(z[8 * c + 4], z[8 * c + 5]), sm100::pack_half2(z[8 * c + 6], z[8 * c + 7]));
        }
        sm100::fence_proxy_async();
        __syncwarp();
        if (lane == 0) {
          if (p < 2)
            sm100::tma_store_2d(&mp.x32out, sw, 64 * cg + 32 * p, m0 + 32 * q);
          else
            sm100::tma_store_2d(&mp.x16out, sw, 64 * cg, m0 + 32 * q);
          sm100::bulk_commit();
        }
      }
#else
      // pass B: x' piece k (rows 32q.., columns 64cg + 16k ..) -> this warp's
      // staging (SW64 fp32 / SW32 fp16, the TMA box layouts) -> TMA stores;
      // the staging is rewritten once the previous piece's stores have read it
      unsigned char* s32 = sStg + ew * (STG32 + STG16);
      unsigned char* s16 = s32 + STG32;
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        float* zk = z + 16 * k;
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          const int col = 64 * cg + 16 * k + 4 * c;
          const float4 g = (*reinterpret_cast<const float4*>(p_g2 + col));
          const float4 be = (*reinterpret_cast<const float4*>(p_be2 + col));
          zk[4 * c] = (zk[4 * c] - mean) * rstd * g.x + be.x;
          zk[4 * c + 1] = (zk[4 * c + 1] - mean) * rstd * g.y + be.y;
          zk[4 * c + 2] = (zk[4 * c + 2] - mean) * rstd * g.z + be.z;
          zk[4 * c + 3] = (zk[4 * c + 3] - mean) * rstd * g.w + be.w;
        }
#if !PREDTOP_L256_STG
        if (lane == 0) sm100::bulk_wait_read0();
#endif
        __syncwarp();
#pragma unroll
        for (int c = 0; c < 4; ++c)
          *reinterpret_cast<float4*>(s32 + lane * 64 + 16 * (c ^ ((lane >> 1) & 3))) =
              make_float4(zk[4 * c], zk[4 * c + 1], zk[4 * c + 2], zk[4 * c + 3]);
#pragma unroll
        for (int c = 0; c < 2; ++c)
          *reinterpret_cast<uint4*>(s16 + lane * 32 + 16 * (c ^ ((lane >> 2) & 1))) =
              make_uint4(sm100::pack_half2(zk[8 * c], zk[8 * c + 1]), sm100::pack_half2(zk[8 * c + 2], zk[8 * c + 3]),
                         sm100::pack_half2(zk[8 * c + 4], zk[8 * c + 5]), sm100::pack_half2(zk[8 * c + 6], zk[8 * c + 7]));
#if PREDTOP_L256_STG
        __syncwarp();
        // read back transposed: fp32 -> lane (row l/4 + 8 rr, 16-byte chunk
        // l%4), fp16 -> (row l/2 + 16 rr, chunk l%2): every store instruction
        // writes whole 64 / 32-byte row segments
#pragma unroll
        for (int rr = 0; rr < 4; ++rr) {
          const int rw = (lane >> 2) + 8 * rr, ch = lane & 3;
          const float4 v = *reinterpret_cast<const float4*>(s32 + rw * 64 + 16 * (ch ^ ((rw >> 1) & 3)));
          if (m0 + 32 * q + rw < args.M)
            *reinterpret_cast<float4*>(args.x32 + (int64_t)(m0 + 32 * q + rw) * D + 64 * cg + 16 * k + 4 * ch) = v;
        }
#pragma unroll
        for (int rr = 0; rr < 2; ++rr) {
          const int rw = (lane >> 1) + 16 * rr, ch = lane & 1;
          const uint4 v = *reinterpret_cast<const uint4*>(s16 + rw * 32 + 16 * (ch ^ ((rw >> 2) & 1)));
          if (m0 + 32 * q + rw < args.M && args.x16 != nullptr)
            *reinterpret_cast<uint4*>(args.x16 + (int64_t)(m0 + 32 * q + rw) * D + 64 * cg + 16 * k + 8 * ch) = v;
        }
        __syncwarp();
#else
        sm100::fence_proxy_async();
        __syncwarp();
        if (lane == 0) {
          sm100::tma_store_2d(&mp.x32out, s32, 64 * cg + 16 * k, m0 + 32 * q);
          if (args.x16 != nullptr) sm100::tma_store_2d(&mp.x16out, s16, 64 * cg + 16 * k, m0 + 32 * q);
          sm100::bulk_commit();
        }
#endif
      }

#endif
      if (leader) LT(i, 11); LW(i, 7);
    }
  }
  if (warp >= 2 && lane == 0) sm100::bulk_wait0();
  __syncwarp();
  sm100::tc_fence_before();
  __syncthreads();
  if (warp == 1) sm100::tmem_dealloc<512>(tmem);
}

}  // namespace

bool layer_tail256_supported(int d, int dff) { return d == D && dff % (2 * FC) == 0 && dff <= kMaxFF; }

predtop_status layer_tail256_launch(const predtop_model_s* m, int l, const __half* att, float* x32, __half* x16,
                                    int M, cudaStream_t st) {
  const int d = m->cfg.d_model, dff = m->cfg.d_ff;
  if (!layer_tail256_supported(d, dff)) {
    set_error("layer tail 256 needs d = 256 and d_ff %% 256 == 0, d_ff <= %d", kMaxFF);
    return PREDTOP_ERR_UNSUPPORTED;
  }
  if (M <= 0) return PREDTOP_OK;
  const LayerDev& L = m->layer[l];
  T256Maps mp;
  if (!encode_tma_2d(&mp.att, att, 2, D, M, 64, 128) || !encode_tma_2d(&mp.x32in, x32, 4, D, M, 32, 128) ||
      !encode_tma_2d(&mp.wo, L.Wo, 2, D, D, 64, 256) || !encode_tma_2d(&mp.w1, L.W1, 2, D, dff, 64, FC) ||
      !encode_tma_2d(&mp.w2, L.W2, 2, dff, D, 64, 256) ||
      !encode_tma_2d(&mp.x32out, x32, 4, D, M, PREDTOP_L256_OUTW ? 32 : 16, 32) ||
      // x16 == nullptr (the last layer: nothing reads the fp16 shadow) skips its stores
      !encode_tma_2d(&mp.x16out, x16 ? (const void*)x16 : (const void*)x32, 2, D, M, PREDTOP_L256_OUTW ? 64 : 16, 32))
    return PREDTOP_ERR_CUDA;
  T256Args a{M, dff, L.bo, L.g1, L.be1, L.b1, L.b2, L.g2, L.be2, m->cfg.ln_eps, x32, x16};
  PT_SMEM_ATTR(k_layer_tail256, SMEM);
  const int sms = num_sms();
  if (!sms) return PREDTOP_ERR_CUDA;
  const int grid = (int)std::min<int64_t>(ceil_div(M, 128), sms);
  k_layer_tail256<<<grid, kThreads, SMEM, st>>>(mp, a);
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

}  // namespace predtop

#ifdef PREDTOP_TRACE
extern "C" PREDTOP_API int predtop_debug_l256_trace(unsigned long long* out) {
  return cudaMemcpyFromSymbol(out, predtop::g_l256, sizeof(predtop::g_l256)) == cudaSuccess ? 0 : -7;
}
extern "C" PREDTOP_API int predtop_debug_l256_trace_w(unsigned long long* out) {
  return cudaMemcpyFromSymbol(out, predtop::g_l256w, sizeof(predtop::g_l256w)) == cudaSuccess ? 0 : -7;
}
#endif
