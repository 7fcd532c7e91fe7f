// layer2.cu -- K7 v2: the post-attention half of the DAG-Transformer layer
// (Fig. 4; reading R6, post-LN encoder layer of [34]),
//     h  = LN1(x + att W_o^T + b_o)
//     x' = LN2(h + ReLU(h W_1^T + b_1) W_2^T + b_2),
// as a persistent tcgen05 kernel with TWO CTAs per SM, so that one CTA's
// LayerNorm / ReLU epilogue overlaps the other CTA's MMAs (the v1 kernel in
// layer.cu runs one 128-row tile per SM and alternates MMA and epilogue).
//
// What makes two CTAs fit (256 TMEM columns, ~102 KB of shared memory each):
//   * TMEM: acc [0,128) holds the O-projection, and after LN1 the epilogue
//     writes h + b_2 back into the same columns (tcgen05.st), so FFN-2
//     accumulates straight onto the residual: acc = h + b_2 + FFN(h), the
//     LN2 input.  acc_f [128,256) is the FFN-1 chunk (128 hidden units),
//     turned in place into the fp16 ReLU output that FFN-2 reads as its A
//     operand from tensor memory (TS-MMA).
//   * Shared memory: a 4-slot ring of 16 KB slices (att K-slices and every
//     weight slice, in MMA consumption order) and the 32 KB fp16 h tile (the
//     FFN-1 A operand).  Each epilogue warp owns one 4 KB piece of the h tile
//     (32 rows x one 64-column K-slice) and reuses it as its private TMA
//     staging buffer: the fp32 residual x comes in as two [32 x 32] boxes,
//     x' (fp32) and its fp16 shadow go out as [32 x 32] / [32 x 64] boxes.
//
// Roles (10 warps): warp 0 TMA producer, warp 1 MMA issuer, warps 2..9
// epilogue (lane quarter q = warp % 4 -> rows 32q.., column half g -> the
// 64 columns [64g, 64g + 64) of the row).
#include <algorithm>

#include "internal.h"
#include "sm100.cuh"

namespace predtop {

#ifdef PREDTOP_TRACE
// Debug timeline of CTA 0 (first 16 tiles): %globaltimer at epilogue phase
// boundaries; MMA-thread wait clocks summed over tiles 2..9 of CTA 0.
__device__ unsigned long long g_tail2_trace[16][16];
__device__ long long g_tail2_mma[8];
__device__ __forceinline__ unsigned long long gtime2() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define T2(i, k)                                                                      \
  do {                                                                                \
    if (leader && blockIdx.x == 0 && (i) < 16) g_tail2_trace[i][k] = gtime2();       \
  } while (0)
#define T2W(k, stmt)                                                                  \
  do {                                                                                \
    const long long t0_ = clock64();                                                  \
    stmt;                                                                             \
    if (blockIdx.x == 0 && i >= 2 && i < 10) g_tail2_mma[k] += clock64() - t0_;      \
  } while (0)
#else
#define T2(i, k) \
  do {           \
  } while (0)
#define T2W(k, stmt) stmt
#endif

namespace {

constexpr int D = 128;           // d_model handled by this kernel
constexpr int FC = 64;           // FFN chunk (hidden units per chunk), two TMEM buffers
constexpr int RS = 4;            // ring slots
constexpr int SLOT = 128 * 128;  // bytes of one [128 rows x 64 fp16] slice
constexpr int SH = 128 * D * 2;  // fp16 h tile (two K-slices)
constexpr int kEpiWarps = 8;
constexpr int kEpi = 32 * kEpiWarps;
constexpr int kThreads = 64 + kEpi;
constexpr int PARAMS = (6 * D + 1024) * 4;
constexpr int SMEM = RS * SLOT + SH + PARAMS + 1024;
constexpr uint32_t TMEM_COLS = 256;
static_assert(SMEM <= 113 * 1024, "two CTAs per SM");

struct Tail2Maps {
  CUtensorMap att, x32, x16, wo, w1, w2, x32in;
};

struct Tail2Args {
  int M, dff;
  const float *bo, *g1, *be1, *b1, *b2, *g2, *be2;
  float eps;
  float* x32;   // residual stream [M][D] fp32 (read, then overwritten with x')
  __half* x16;  // its fp16 shadow [M][D]
};

// Residual I/O of the epilogue.  2 (default): the producer streams the x tile
// through the ring (4 slots of [128 rows x 32 fp32], right after the tile's
// att / W_o slices), so it arrives while the previous tile finishes; x' goes
// out through the warp's 4 KB staging piece by TMA.  1: x also comes in
// through the staging piece, two [32 x 32] boxes after the previous tile's
// stores have drained (~3 us per tile exposed).  0 selects plain 16-byte global
// loads/stores straight between registers and memory (each thread owns 64
// contiguous columns of one row); measured 2x slower on 1xB200 (lanes 512 B
// apart: 32 sectors per instruction, LSU-bound; tools/tail2_trace.py), kept
// for reference.
#ifndef PREDTOP_TAIL2_TMA_IO
#define PREDTOP_TAIL2_TMA_IO 2
#endif

__device__ __forceinline__ void tma_prefetch_l2_2d(const CUtensorMap* map, int32_t c0, int32_t c1) {
  asm volatile("cp.async.bulk.prefetch.tensor.2d.L2.global [%0, {%1, %2}];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(c0), "r"(c1)
               : "memory");
}

// 16 fp32 columns registers -> TMEM (32x32b.x16)
__device__ __forceinline__ void tmem_st_f16(uint32_t taddr, const float* v) {
  uint32_t r[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) r[i] = __float_as_uint(v[i]);
  sm100::tmem_st16(taddr, r);
}

__global__ void __launch_bounds__(kThreads, 2) k_layer_tail2(const __grid_constant__ Tail2Maps mp, Tail2Args args) {
  extern __shared__ unsigned char dsm[];
  unsigned char* base = sm100::align1024(dsm);
  unsigned char* ring = base;               // RS x 16 KB
  unsigned char* sH = ring + RS * SLOT;     // [2 K-slices][128 rows x 64] fp16, SW128
  float* sPar = reinterpret_cast<float*>(sH + SH);
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
  __shared__ __align__(8) uint64_t f_full[2], p_ready[2];  // per acc_f buffer
  __shared__ __align__(8) uint64_t xbar[kEpiWarps];
  __shared__ uint32_t tmem_slot;
  __shared__ float red[2][2][128];

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ntiles = (int)ceil_div(args.M, 128);
  const int NJ = args.dff / FC;

  if (threadIdx.x == 0) {
    for (int s = 0; s < RS; ++s) {
      sm100::mbar_init(&ring_full[s], 1);
      sm100::mbar_init(&ring_empty[s], 1);
    }
    uint64_t* singles[] = {&o_full, &o_empty, &h_ready, &out_full, &f_full[0], &f_full[1]};
    for (uint64_t* b : singles) sm100::mbar_init(b, 1);
    sm100::mbar_init(&p_ready[0], kEpiWarps);  // one arrival per epilogue warp
    sm100::mbar_init(&p_ready[1], kEpiWarps);
    for (int w = 0; w < kEpiWarps; ++w) sm100::mbar_init(&xbar[w], 1);
    sm100::fence_mbar_init();
  }
  if (warp == 1) sm100::tmem_alloc<TMEM_COLS>(&tmem_slot);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem = tmem_slot;
  // TMEM: acc [0, 128) O-projection, then h + b_2 + FFN(h); acc_f buffers
  // [128, 192) and [192, 256): FFN-1 chunk j in buffer j & 1
  const uint32_t acc = tmem, acc_f = tmem + D;

  if (warp == 0) {
    if (lane == 0) {  // ------------------------------------------ TMA producer
      sm100::tma_prefetch(&mp.att);
      sm100::tma_prefetch(&mp.x32);
      sm100::tma_prefetch(&mp.wo);
      sm100::tma_prefetch(&mp.w1);
      sm100::tma_prefetch(&mp.w2);
      int it = 0;
      auto load = [&](const CUtensorMap* m, int c0, int c1) {
        const int s = it % RS;
        sm100::mbar_wait(&ring_empty[s], ((it / RS) & 1) ^ 1);
        sm100::mbar_arrive_expect_tx(&ring_full[s], SLOT);
        sm100::tma_load_2d(ring + s * SLOT, m, &ring_full[s], c0, c1);
        ++it;
      };
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const int m0 = t * 128;
        const int tn = t + gridDim.x;
        if (tn < ntiles)  // the next tile's residual: into L2 while this tile runs
          for (int b = 0; b < D / 32; ++b) tma_prefetch_l2_2d(&mp.x32, b * 32, tn * 128);
        for (int kc = 0; kc < D / 64; ++kc) {
          load(&mp.att, kc * 64, m0);
          load(&mp.wo, kc * 64, 0);
        }
#if PREDTOP_TAIL2_TMA_IO == 2
        // the residual x tile for the epilogue: 4 slots of [128 rows x 32 fp32]
        // (SW128), after this tile's att/W_o (so the O-projection never waits
        // for them) and before its FFN weights
        for (int k = 0; k < D / 32; ++k) load(&mp.x32in, k * 32, m0);
#endif
        // W_1 chunk j: one slot, two [64 x 64] K-slices; W_2 chunk j: one
        // [128 x 64] slot.  Order = MMA order: F1_0 F1_1 F2_0 F1_2 F2_1 ...
        auto load_w1 = [&](int j) {
          const int s = it % RS;
          sm100::mbar_wait(&ring_empty[s], ((it / RS) & 1) ^ 1);
          sm100::mbar_arrive_expect_tx(&ring_full[s], SLOT);
          for (int kc = 0; kc < D / 64; ++kc)
            sm100::tma_load_2d(ring + s * SLOT + kc * (FC * 128), &mp.w1, &ring_full[s], kc * 64, j * FC);
          ++it;
        };
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
      int it = 0;
      int i = 0;
      auto slot_wait = [&]() -> uint32_t {
        const int s = it % RS;
        T2W(0, sm100::mbar_wait(&ring_full[s], (it / RS) & 1));
        sm100::tc_fence_after();
        return sm100::smem_u32(ring + s * SLOT);
      };
      auto slot_free = [&]() {
        sm100::mma_commit(&ring_empty[it % RS]);
        ++it;
      };
      const uint32_t aH = sm100::smem_u32(sH);
      for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
#ifdef PREDTOP_TRACE
        const long long tile_t0 = clock64();
#endif
        // ---- O-projection: acc = att W_o^T (acc free once LN2 of the previous tile read it)
        T2W(1, sm100::mbar_wait(&o_empty, (i & 1) ^ 1));
        sm100::tc_fence_after();
        for (int kc = 0; kc < D / 64; ++kc) {
          const uint32_t a0 = slot_wait();
          const int sa = it % RS;
          ++it;
          const uint32_t b0 = slot_wait();
#pragma unroll
          for (int kk = 0; kk < 4; ++kk)
            sm100::mma_f16_ss(acc, sm100::make_sdesc<128>(a0 + kk * 32), sm100::make_sdesc<128>(b0 + kk * 32),
                              id_N128, (kc | kk) != 0);
          sm100::mma_commit(&ring_empty[sa]);
          slot_free();
        }
        sm100::mma_commit(&o_full);
#if PREDTOP_TAIL2_TMA_IO == 2
        // the x slots belong to the epilogue.  Skipping them is safe: the next
        // slot_wait (FFN-1, after h_ready) is on a phase whose predecessor
        // (the x load) the epilogue consumed before h_ready
        it += D / 32;
#endif
        // ---- FFN: acc already holds h + b_2 (written by the epilogue after LN1)
        T2W(2, sm100::mbar_wait(&h_ready, i & 1));
        sm100::tc_fence_after();
        constexpr uint32_t id_N64 = sm100::make_idesc_f16(128, FC);
        // FFN-1 chunk j -> acc_f buffer j & 1.  Chunk j+2 reuses the buffer
        // whose P FFN-2 chunk j (issued just before by this thread) reads:
        // tcgen05.mma of one thread executes in issue order.
        auto ffn1 = [&](int j) {
          const uint32_t b0 = slot_wait();
          const uint32_t dst = acc_f + (uint32_t)((j & 1) * FC);
#pragma unroll
          for (int kc = 0; kc < D / 64; ++kc)
#pragma unroll
            for (int kk = 0; kk < 4; ++kk)
              sm100::mma_f16_ss(dst, sm100::make_sdesc<128>(aH + kc * SLOT + kk * 32),
                                sm100::make_sdesc<128>(b0 + kc * (FC * 128) + kk * 32), id_N64, (kc | kk) != 0);
          slot_free();
          sm100::mma_commit(&f_full[j & 1]);
        };
        ffn1(0);
        for (int j = 0; j < NJ; ++j) {
          if (j + 1 < NJ) ffn1(j + 1);  // keeps the tensor pipe busy during ReLU_j
          // FFN-2 chunk j: acc += P_j W_2[:, chunk]^T, P_j from TMEM: epilogue
          // warp g leaves hidden units [32g, 32g + 32) as 16 packed fp16
          // columns at 32g of the buffer, so K-step ks sits at 32(ks/2) + 8(ks%2).
          T2W(3, sm100::mbar_wait(&p_ready[j & 1], ((i * NJ + j) >> 1) & 1));
          sm100::tc_fence_after();
          const uint32_t b0 = slot_wait();
          const uint32_t src = acc_f + (uint32_t)((j & 1) * FC);
#pragma unroll
          for (int ks = 0; ks < FC / 16; ++ks)
            sm100::mma_f16_ts(acc, src + (uint32_t)(32 * (ks / 2) + 8 * (ks % 2)),
                              sm100::make_sdesc<128>(b0 + ks * 32), id_N128, 1u);
          slot_free();
        }
        sm100::mma_commit(&out_full);
#ifdef PREDTOP_TRACE
        if (blockIdx.x == 0 && i >= 2 && i < 10) g_tail2_mma[4] += clock64() - tile_t0;
#endif
      }
    }
  } else {
    // ------------------------------------------ epilogue warps 2..9
    const int ew = warp - 2;
    const int q = warp & 3, g = ew >> 2;
    const int r = q * 32 + lane;  // tile row of this thread (TMEM lane)
    const uint32_t lrow = (uint32_t)(q * 32) << 16;
    const bool leader = (ew == 0 && lane == 0);
    // this warp's 4 KB piece of the h tile: rows 32q.. of K-slice g (SW128)
    unsigned char* stg = sH + g * SLOT + q * 4096;
#if PREDTOP_TAIL2_TMA_IO == 1
    uint64_t* xb = &xbar[ew];
    uint32_t xphase = 0;
    auto x_load = [&](int m0, int k) {  // [32 rows x 32 fp32] box of the residual
      if (lane == 0) {
        sm100::mbar_arrive_expect_tx(xb, 4096);
        sm100::tma_load_2d(stg, &mp.x32, xb, 64 * g + 32 * k, m0 + 32 * q);
      }
    };
#endif
    auto stage_f32 = [&](const float* v) {  // 32 fp32 of row `lane` -> staging (SW128)
#pragma unroll
      for (int c = 0; c < 8; ++c)
        *reinterpret_cast<float4*>(stg + sm100::swz<128>(lane, c)) =
            make_float4(v[4 * c], v[4 * c + 1], v[4 * c + 2], v[4 * c + 3]);
    };
    auto store_wait = [&]() {  // staging may be rewritten once the bulk store has read it
      if (lane == 0) sm100::bulk_wait_read0();
      __syncwarp();
    };
    // Cross-group LayerNorm statistic of row r: s -> sum over both column halves.
    auto row_sum = [&](float s, int which) {
      red[which][g][r] = s;
      sm100::named_bar<kEpi>(1);
      return red[which][0][r] + red[which][1][r];
    };
    float x[64];
    int i = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
      const int m0 = t * 128;
      const int cbase = i * NJ;
      T2(i, 0);
      // ---- residual x (fp32) -> registers
#if PREDTOP_TAIL2_TMA_IO == 2
      // from the ring: slots (xit + 2g + k) % RS hold columns [64g + 32k, +32).
      // o_full first: the O-projection consumed this tile's att / W_o, i.e.
      // the previous phase of each x slot completed, so the parity wait below
      // is never two phases ahead (it would alias and return at once)
      sm100::mbar_wait(&o_full, i & 1);
      const int xit = i * (2 * (D / 64) + D / 32 + 2 * NJ) + 2 * (D / 64);
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        const int itk = xit + 2 * g + k;
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
      sm100::fence_proxy_async();  // these generic reads before the slots' next TMA writes
#elif !PREDTOP_TAIL2_TMA_IO
      {
        const int row = m0 + r;
        const float4* src = reinterpret_cast<const float4*>(args.x32 + (int64_t)row * D + 64 * g);
#pragma unroll
        for (int c = 0; c < 16; ++c) {
          const float4 v = row < args.M ? __ldcg(src + c) : make_float4(0.f, 0.f, 0.f, 0.f);
          x[4 * c] = v.x;
          x[4 * c + 1] = v.y;
          x[4 * c + 2] = v.z;
          x[4 * c + 3] = v.w;
        }
      }
#else
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        store_wait();
        x_load(m0, k);
        sm100::mbar_wait(xb, xphase);
        xphase ^= 1u;
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          const float4 v = *reinterpret_cast<const float4*>(stg + sm100::swz<128>(lane, c));
          x[32 * k + 4 * c] = v.x;
          x[32 * k + 4 * c + 1] = v.y;
          x[32 * k + 4 * c + 2] = v.z;
          x[32 * k + 4 * c + 3] = v.w;
        }
        // WAR across proxies: this lane's generic reads of the piece are
        // ordered before the next TMA write into it (issued by lane 0 after
        // the __syncwarp in store_wait)
        sm100::fence_proxy_async();
      }
#endif
      __syncwarp();
      T2(i, 1);
      // ---- LN1: z = x + acc + b_o
      sm100::mbar_wait(&o_full, i & 1);
      sm100::tc_fence_after();
      T2(i, 2);
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
#if PREDTOP_TAIL2_TMA_IO == 2
        if (leader)  // every epilogue thread has read its x (the row_sum barrier): free the x slots
          for (int k = 0; k < D / 32; ++k) sm100::mbar_arrive(&ring_empty[(xit + k) % RS]);
#endif
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
#if PREDTOP_TAIL2_TMA_IO == 2
      store_wait();  // the previous tile's x16 store has read the staging piece
#endif
      // h (fp16) -> the FFN-1 A operand; h + b_2 -> acc (FFN-2 accumulates onto it)
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
        tmem_st_f16(acc + lrow + 64 * g + 16 * k, hb);
      }
      sm100::tmem_wait_st();
      sm100::fence_proxy_async();
      sm100::tc_fence_before();
      sm100::named_bar<kEpi>(1);
      if (leader) sm100::mbar_arrive(&h_ready);
      T2(i, 3);
      // ---- FFN chunks: ReLU(acc_f + b_1) -> fp16 pairs back into acc_f
      for (int j = 0; j < NJ; ++j) {
        const int cj = cbase + j;
        sm100::mbar_wait(&f_full[j & 1], (cj >> 1) & 1);
        sm100::tc_fence_after();
        if (j < 4) T2(i, 4 + j);
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
        if (lane == 0) sm100::mbar_arrive(&p_ready[j & 1]);  // this warp's part of P_j is in TMEM
        if (j < 4) T2(i, 8 + j);
      }
      // ---- LN2: z = acc (= h + b_2 + FFN(h))
      sm100::mbar_wait(&out_full, i & 1);
      sm100::tc_fence_after();
      T2(i, 12);
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
      T2(i, 13);
#if !PREDTOP_TAIL2_TMA_IO
      // ---- x' (fp32) and its fp16 shadow, straight from registers
      if (m0 + r < args.M) {
        float4* d32 = reinterpret_cast<float4*>(args.x32 + (int64_t)(m0 + r) * D + 64 * g);
        uint4* d16 = reinterpret_cast<uint4*>(args.x16 + (int64_t)(m0 + r) * D + 64 * g);
#pragma unroll
        for (int c = 0; c < 16; ++c) d32[c] = make_float4(x[4 * c], x[4 * c + 1], x[4 * c + 2], x[4 * c + 3]);
#pragma unroll
        for (int c = 0; c < 8; ++c)
          d16[c] = make_uint4(sm100::pack_half2(x[8 * c], x[8 * c + 1]), sm100::pack_half2(x[8 * c + 2], x[8 * c + 3]),
                              sm100::pack_half2(x[8 * c + 4], x[8 * c + 5]), sm100::pack_half2(x[8 * c + 6], x[8 * c + 7]));
      }
#else
      // ---- x' (fp32, two boxes) and its fp16 shadow through the staging piece.
      // The piece held h, read by FFN-1 MMAs that completed before out_full.
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        if (k) store_wait();
        stage_f32(x + 32 * k);
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
#endif
      T2(i, 14);
    }
    if (lane == 0) sm100::bulk_wait0();
  }
  __syncwarp();
  sm100::tc_fence_before();
  __syncthreads();
  if (warp == 1) sm100::tmem_dealloc<TMEM_COLS>(tmem);
}


}  // namespace

bool layer_tail2_supported(int d, int dff) { return d == D && dff % (2 * FC) == 0 && dff <= 1024; }  // even chunk count (buffer phases)

predtop_status layer_tail2_launch(const predtop_model_s* m, int l, const __half* att, float* x32,
                                  __half* x16, int M, cudaStream_t st) {
  const int d = m->cfg.d_model, dff = m->cfg.d_ff;
  if (!layer_tail2_supported(d, dff)) {
    set_error("layer tail v2 needs d = 128 and d_ff %% 128 == 0");
    return PREDTOP_ERR_UNSUPPORTED;
  }
  if (M <= 0) return PREDTOP_OK;
  const LayerDev& L = m->layer[l];
  Tail2Maps mp;
  if (!encode_tma_2d(&mp.att, att, 2, d, M, 64, 128) || !encode_tma_2d(&mp.x32, x32, 4, d, M, 32, 32) ||
      !encode_tma_2d(&mp.x16, x16, 2, d, M, 64, 32) || !encode_tma_2d(&mp.x32in, x32, 4, d, M, 32, 128))
    return PREDTOP_ERR_CUDA;
  mp.wo = L.tm_o;
  mp.w1 = L.tm_1h;
  mp.w2 = L.tm_2;
  Tail2Args a{M, dff, L.bo, L.g1, L.be1, L.b1, L.b2, L.g2, L.be2, m->cfg.ln_eps, x32, x16};
  PT_SMEM_ATTR(k_layer_tail2, SMEM);
  const int g_sms2 = num_sms();
  if (!g_sms2) return PREDTOP_ERR_CUDA;
  const int grid = (int)std::min<int64_t>(ceil_div(M, 128), 2 * g_sms2);
  k_layer_tail2<<<grid, kThreads, SMEM, st>>>(mp, a);
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

}  // namespace predtop

#ifdef PREDTOP_TRACE
extern "C" PREDTOP_API int predtop_debug_tail2_trace(unsigned long long* out) {
  if (cudaMemcpyFromSymbol(out, predtop::g_tail2_trace, sizeof(predtop::g_tail2_trace)) != cudaSuccess) return -7;
  return cudaMemcpyFromSymbol(out + 256, predtop::g_tail2_mma, sizeof(predtop::g_tail2_mma)) == cudaSuccess ? 0 : -7;
}
#endif
