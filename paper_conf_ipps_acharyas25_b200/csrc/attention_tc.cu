// attention_tc.cu -- K6 on the 5th-generation tensor cores (d_h = 16):
// reachability-masked multi-head attention, Eqn 1, reading R1,
//     O_h = softmax(Q_h K_h^T / sqrt(d_h) + M) V_h,  M(u,v) = 0 iff bit M[u][v]
//     of M = R | R^T | I is set (DAGRA), else -inf.
//
// One CTA = one (graph, 128-row query tile, head).  Every query row is one
// TMEM lane, so a softmax thread owns a whole row: no shuffles, 32
// independent exponentials per 32-key chunk.
//
//   warp 0      TMA: the Q tile (128 x 16) and all K rows of the graph
//               (SWIZZLE_32B, the UMMA K-major layout for K = 16)
//   warp 1      TMEM owner + MMA issuer (one thread):
//                 S_c   = Q K_c^T        tcgen05.mma SS, M=128 N=32 K=16
//                 O    += P_c [V_c | 1]  tcgen05.mma TS, A = P_c from TMEM,
//                                        N=32 (16 value + 16 ones columns:
//                                        the row sums l come out of the MMA)
//   warps 2..5  softmax (row = TMEM lane): mask, exp2, P -> TMEM as fp16;
//               before the loop they transpose V into the K-major
//               [V_c | 1]^T operand (SWIZZLE_64B), after it normalise O.
//
// TMEM (128 columns): S0 [0,32) | S1 [32,64) | P0 [64,80) | P1 [80,96) |
// O [96,128).  S and P are double buffered so QK^T of chunk c+2 overlaps the
// softmax of chunk c+1.  The softmax warps pre-set S_c to -m (tcgen05.st), so
// the QK^T MMA accumulates s - m directly.
//
// Online softmax in log2 units (Q pre-scaled by log2(e)/sqrt(d_h) in the QKV
// epilogue).  The reference m of a row starts at its diagonal score (always
// allowed: M includes I, so the row max is >= it) and only moves when a
// score exceeds it by more than 8, so P = exp2(s - m) <= 256 stays exact in
// fp16 (lazy rescaling: O and l are rescaled in TMEM, rarely).
#include <algorithm>

#include "internal.h"
#include "sm100.cuh"

namespace predtop {

namespace {

constexpr int kRows = 128;   // query rows per CTA (TMEM lanes)
constexpr int kKeys = 32;    // keys per chunk (S columns)
constexpr int kDh = 16;
constexpr int kThreads = 192;
constexpr int kQBytes = kRows * kDh * 2;     // 4 KB, SW32
constexpr int kVtBytes = 2 * 16 * kKeys * 2; // [V_c | 1]^T: 32 rows x 64 B, SW64
#ifndef PREDTOP_ATTN_POLY
#define PREDTOP_ATTN_POLY 12
#endif
constexpr int kPoly = PREDTOP_ATTN_POLY;     // keys per chunk whose exp2 runs on the FMA pipe
static_assert(kPoly % 2 == 0 && kPoly <= kKeys, "kPoly");

// exp2 of two arguments in (-inf, 8] on the FMA pipe (packed f32x2), as the
// fp16 pair the PV MMA consumes: x = max(x, -126); j = rint(x) (magic-number
// add); 2^(x-j) by a degree-3 minimax polynomial on [-1/2, 1/2] (max rel.
// error 7.5e-5, below the fp16 rounding of P); 2^j added to the exponent.
__device__ __forceinline__ uint32_t exp2_poly2(float x0, float x1) {
  x0 = fmaxf(x0, -126.f);
  x1 = fmaxf(x1, -126.f);
  uint64_t x, t, jj, f, p;
  asm("mov.b64 %0, {%1, %2};" : "=l"(x) : "f"(x0), "f"(x1));
  const uint64_t magic = 0x4B4000004B400000ull;  // 1.5 * 2^23, twice
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(t) : "l"(x), "l"(magic));
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(jj) : "l"(t), "l"(magic));
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(f) : "l"(x), "l"(jj));
  const uint64_t c3 = 0x3D61FBAF3D61FBAFull;  // 0.0551716648
  const uint64_t c2 = 0x3E786F0D3E786F0Dull;  // 0.2426111251
  const uint64_t c1 = 0x3F31798D3F31798Dull;  // 0.6932609677
  const uint64_t c0 = 0x3F7FFB493F7FFB49ull;  // 0.9999280572
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(p) : "l"(c3), "l"(f), "l"(c2));
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(p) : "l"(p), "l"(f), "l"(c1));
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(p) : "l"(p), "l"(f), "l"(c0));
  uint32_t p0, p1, t0, t1;
  asm("mov.b64 {%0, %1}, %2;" : "=r"(p0), "=r"(p1) : "l"(p));
  asm("mov.b64 {%0, %1}, %2;" : "=r"(t0), "=r"(t1) : "l"(t));
  // t = 1.5 * 2^23 + j: its low bits are j; (t << 23) wraps to j << 23
  const float y0 = __uint_as_float(p0 + (t0 << 23)), y1 = __uint_as_float(p1 + (t1 << 23));
  return sm100::pack_half2(y0, y1);
}

#ifdef PREDTOP_TRACE
// debug timeline of one CTA: %globaltimer at pipeline events
__device__ unsigned long long g_at[6][16];
__device__ __forceinline__ unsigned long long at_now() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define ATR(k, i) \
  do {            \
    if (blockIdx.x == 8000 && (i) < 16) g_at[k][i] = at_now(); \
  } while (0)
#else
#define ATR(k, i) \
  do {            \
  } while (0)
#endif

#ifdef PREDTOP_SPIN_WAIT
#define WAIT sm100::mbar_wait
#else
#define WAIT sm100::mbar_wait_sleep
#endif

__device__ __forceinline__ float ex2f(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

__global__ void __launch_bounds__(kThreads, 4)
    k_attn_tc(const __grid_constant__ CUtensorMap tq, DagDev d, int G, int H, int dmodel,
              const __half* __restrict__ qkv, __half* __restrict__ out, int krows_cap) {
  extern __shared__ unsigned char dsm[];
  unsigned char* base = sm100::align1024(dsm);
  unsigned char* sQ = base;                   // [128][16] fp16, SW32
  unsigned char* sK = sQ + kQBytes;           // [krows_cap][16] fp16, SW32
  unsigned char* sVs = sK + krows_cap * 32;   // [krows_cap][16] fp16, SW32 (V staging)
  unsigned char* sQm = sVs + krows_cap * 32;  // 2 x [128][16] fp16 SW32: col 0 = -m (per S buffer)
  unsigned char* sOne = sQm + 2 * kQBytes;    // [32][16] fp16 SW32: col 0 = 1
  unsigned char* sVt = sOne + 1024;           // per chunk: [V_c | 1]^T, SW64 (1 KB aligned)
  __shared__ __align__(8) uint64_t bar_ld, vt_ready, s_full[2], p_ready[2], pv_done, o_full;
  __shared__ uint32_t tmem_slot;

  const int h = blockIdx.x % H;
  const int widx = blockIdx.x / H;
  if (widx >= d.qtile_off[G]) return;
  const int2 wk = d.work[widx];
  const int g = wk.x, qt = wk.y;
  if ((unsigned)g >= (unsigned)G || d.status[g] != PREDTOP_OK) return;
  const int64_t n0 = d.node_ptr[g];
  const int N = (int)(d.node_ptr[g + 1] - n0);
  const int W = 2 * ((N + 127) / 128);
  const int nch = (N + kKeys - 1) / kKeys;
  const int krows = ((N + 127) / 128) * 128;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    sm100::mbar_init(&bar_ld, 1);
    sm100::mbar_init(&vt_ready, 1);
    sm100::mbar_init(&s_full[0], 1);
    sm100::mbar_init(&s_full[1], 1);
    sm100::mbar_init(&p_ready[0], 4);
    sm100::mbar_init(&p_ready[1], 4);
    sm100::mbar_init(&pv_done, 1);
    sm100::mbar_init(&o_full, 1);
    sm100::fence_mbar_init();
  }
  if (warp == 1) sm100::tmem_alloc<128>(&tmem_slot);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem = tmem_slot;
  const uint32_t tP = tmem + 64;  // P0 [64,80) | P1 [80,96): fp16 pairs
  const uint32_t tO = tmem + 96;

  if (warp == 0) {
    if (lane == 0) {  // ------------------------------------------ TMA
      sm100::mbar_arrive_expect_tx(&bar_ld, (uint32_t)(kQBytes + 2 * krows * 32));
      sm100::tma_load_2d(sQ, &tq, &bar_ld, h * kDh, (int)(n0 + qt * kRows));
      for (int r = 0; r < krows; r += 128) {
        sm100::tma_load_2d(sK + r * 32, &tq, &bar_ld, dmodel + h * kDh, (int)(n0 + r));
        sm100::tma_load_2d(sVs + r * 32, &tq, &bar_ld, 2 * dmodel + h * kDh, (int)(n0 + r));
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {  // ------------------------------------------ MMA issuer
      constexpr uint32_t idesc = sm100::make_idesc_f16(128, 32);
      const uint32_t aQ = sm100::smem_u32(sQ), aK = sm100::smem_u32(sK), aV = sm100::smem_u32(sVt);
      const uint32_t aQm = sm100::smem_u32(sQm), aOne = sm100::smem_u32(sOne);
      // S_c = Q K_c^T + Qm_b 1^T = q.k - m  (Qm_b: column 0 = -m per row)
      auto qk = [&](int c) {
        const uint32_t tS = tmem + 32 * (c & 1);
        sm100::mma_f16_ss(tS, sm100::make_sdesc<32>(aQ), sm100::make_sdesc<32>(aK + c * 1024), idesc, 0u);
        sm100::mma_f16_ss(tS, sm100::make_sdesc<32>(aQm + (c & 1) * kQBytes), sm100::make_sdesc<32>(aOne), idesc, 1u);
        sm100::mma_commit(&s_full[c & 1]);
      };
      ATR(0, 0);
      WAIT(&bar_ld, 0);
      ATR(0, 1);
      WAIT(&vt_ready, 0);
      ATR(0, 2);
      sm100::tc_fence_after();
      qk(0);
      if (nch > 1) qk(1);
      for (int c = 0; c < nch; ++c) {
        WAIT(&p_ready[c & 1], (c >> 1) & 1);
        ATR(1, c);
        sm100::tc_fence_after();
#pragma unroll
        for (int kk = 0; kk < 2; ++kk)
          sm100::mma_f16_ts(tO, tP + 16 * (c & 1) + 8 * kk, sm100::make_sdesc<64>(aV + c * kVtBytes + kk * 32),
                            idesc, (c > 0 || kk > 0) ? 1u : 0u);
        sm100::mma_commit(&pv_done);
        // p_ready(c): S_{c&1} was read and Qm_{c&1} holds the current -m
        if (c + 2 < nch) qk(c + 2);
      }
      sm100::mma_commit(&o_full);
    }
  } else {
    // ------------------------------------------------------------ softmax
    const int t = threadIdx.x - 64;  // 0..127
    const int q4 = warp & 3;
    const int r = 32 * q4 + lane;  // TMEM lane = row of the q-tile
    const int row = qt * kRows + r;
    const bool valid = row < N;
    const bool warp_dead = qt * kRows + 32 * q4 >= N;
    const uint32_t lrow = (uint32_t)(32 * q4) << 16;
    // (0) the mask word of this row and the Q/K/V tiles (TMA)
    const uint64_t* Mrow = d.M + d.row_off[g] + (int64_t)(valid ? row : 0) * W;
    uint64_t mw_raw = valid ? Mrow[0] : 0ull, mw = 0ull;  // stored layout -> mask_unperm at use
    WAIT(&bar_ld, 0);
    // (1) reference m: the diagonal score q_row . k_row (fp32, from the SW32
    // tiles: 16-byte chunk j of row x sits at x*32 + 16*(j ^ ((x >> 2) & 1))),
    // rounded to fp16 (it enters the MMA as an fp16 operand; every use below
    // takes the same rounded value).  Qm_0 = Qm_1 = [-m 0 ... 0], 1 = [1 0 ... 0].
    float m = 0.f;
    if (valid) {
      const int kr = qt * kRows + r;  // the row's own key
#pragma unroll
      for (int j = 0; j < 2; ++j) {
        const uint4 a = *reinterpret_cast<const uint4*>(sQ + r * 32 + 16 * (j ^ ((r >> 2) & 1)));
        const uint4 bq = *reinterpret_cast<const uint4*>(sK + kr * 32 + 16 * (j ^ ((kr >> 2) & 1)));
        const uint32_t aw[4] = {a.x, a.y, a.z, a.w}, bw[4] = {bq.x, bq.y, bq.z, bq.w};
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const float2 x = __half22float2(*reinterpret_cast<const __half2*>(&aw[i]));
          const float2 y = __half22float2(*reinterpret_cast<const __half2*>(&bw[i]));
          m += x.x * y.x + x.y * y.y;
        }
      }
    }
    m = __half2float(__float2half_rn(m));
    {
      const uint32_t nm = (uint32_t)__half_as_ushort(__float2half_rn(-m));
      const int c0 = 16 * ((r >> 2) & 1), c1 = 16 - c0;
#pragma unroll
      for (int b = 0; b < 2; ++b) {
        unsigned char* q = sQm + b * kQBytes + r * 32;
        *reinterpret_cast<uint4*>(q + c0) = make_uint4(nm, 0u, 0u, 0u);
        *reinterpret_cast<uint4*>(q + c1) = make_uint4(0u, 0u, 0u, 0u);
      }
      if (t < 32) {
        const int o0 = 16 * ((t >> 2) & 1);
        *reinterpret_cast<uint4*>(sOne + t * 32 + o0) = make_uint4(0x3C00u, 0u, 0u, 0u);
        *reinterpret_cast<uint4*>(sOne + t * 32 + 16 - o0) = make_uint4(0u, 0u, 0u, 0u);
      }
    }
    // (2) [V_c | 1]^T for every chunk (rows j < 16: column j of V; rows
    // 16..31: ones), K-major SW64: element (j, key k) at swz64(j, k/8) + 2(k%8).
    // One warp-step = 16 keys: ldmatrix.x4.trans of the SW32 V staging tile
    // (lanes 0-7: keys k0..k0+7 cols 0-7, 8-15: cols 8-15, 16-31: keys +8)
    // gives lane L the key pair (2(L%4), +1) of column L/4 (+8) in each reg.
    {
      const uint32_t vs = sm100::smem_u32(sVs);
      for (int k0 = 16 * (warp - 2); k0 < nch * kKeys; k0 += 64) {
        const int key = k0 + (lane & 7) + 8 * (lane >> 4), j = (lane >> 3) & 1;
        uint32_t v0, v1, v2, v3;
        asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
                     : "=r"(v0), "=r"(v1), "=r"(v2), "=r"(v3)
                     : "r"(vs + key * 32 + 16 * (j ^ ((key >> 2) & 1))));
        unsigned char* tile = sVt + (k0 / kKeys) * kVtBytes;
        const int kc = k0 % kKeys, col = lane >> 2, kp = 2 * (lane & 3);
        *reinterpret_cast<uint32_t*>(tile + sm100::swz<64>(col, kc >> 3) + 2 * kp) = v0;
        *reinterpret_cast<uint32_t*>(tile + sm100::swz<64>(col + 8, kc >> 3) + 2 * kp) = v1;
        *reinterpret_cast<uint32_t*>(tile + sm100::swz<64>(col, (kc + 8) >> 3) + 2 * kp) = v2;
        *reinterpret_cast<uint32_t*>(tile + sm100::swz<64>(col + 8, (kc + 8) >> 3) + 2 * kp) = v3;
      }
      for (int i = t; i < nch * 64; i += 128) {  // ones: 1 KB (64 x 16 B) per chunk
        unsigned char* tile = sVt + (i >> 6) * kVtBytes + 1024;
        *reinterpret_cast<uint4*>(tile + (i & 63) * 16) = make_uint4(0x3C003C00u, 0x3C003C00u, 0x3C003C00u, 0x3C003C00u);
      }
      sm100::fence_proxy_async();
      sm100::named_bar<128>(1);
      if (t == 0) sm100::mbar_arrive(&vt_ready);
      if (t == 0) ATR(0, 5);
    }
    // (3) chunks.  S_b = q.k - mu_b where mu_b is the m written to Qm_b when
    // its QK^T was issued; a row whose m moved since corrects by (m - mu_b)
    // (rare).  Warps whose 32 rows are all past N only keep the p_ready
    // count; chunks with no allowed pair in the warp's rows store P = 0.
    // Exponentials: MUFU ex2 for keys [0, 32 - kPoly), the FMA-pipe
    // polynomial (exp2_poly2) for the last kPoly keys of each chunk.
    float mu0 = m, mu1 = m;
    auto chunk = [&](int c, int b) {
      if (!b) mw = mask_unperm(mw_raw);
      const uint32_t bits = b ? (uint32_t)(mw >> 32) : (uint32_t)mw;
      if (b && valid && c + 1 < nch) mw_raw = Mrow[(c + 1) >> 1];
      if (warp == 2 && lane == 0) ATR(2, c);
      WAIT(&s_full[b], (c >> 1) & 1);
      if (warp == 2 && lane == 0) ATR(3, c);
      sm100::tc_fence_after();
      if (warp_dead) {
        __syncwarp();
        if (lane == 0) sm100::mbar_arrive(&p_ready[b]);
        return;
      }
      const uint32_t tS = tmem + 32 * b + lrow;
      uint32_t p[kKeys / 2];
      float& mu = b ? mu1 : mu0;
      if (__any_sync(0xffffffffu, bits != 0u)) {
        float s[kKeys];
        sm100::tmem_ld<kKeys>(tS, s);
        const float fix = m - mu;
        if (__any_sync(0xffffffffu, fix != 0.f)) {
#pragma unroll
          for (int k = 0; k < kKeys; ++k) s[k] -= fix;
        }
        float mx = -INFINITY;
#pragma unroll
        for (int k = 0; k < kKeys; ++k) {
          s[k] = ((bits >> k) & 1u) ? s[k] : -INFINITY;
          mx = fmaxf(mx, s[k]);
        }
        if (__any_sync(0xffffffffu, mx > 8.f)) {
          // rare: move m to the new maximum (fp16-rounded), rescale O and l
          // (TMEM) once the previous PV (the last writer of O) has completed
          const float mn = mx > 8.f ? __half2float(__float2half_rn(m + mx)) : m;
          const float dl = mn - m;
          m = mn;
#pragma unroll
          for (int k = 0; k < kKeys; ++k) s[k] -= dl;
          if (c > 0) {
            WAIT(&pv_done, (c - 1) & 1);
            sm100::tc_fence_after();
            const float al = ex2f(-dl);
#pragma unroll 1
            for (int hf = 0; hf < 2; ++hf) {
              float o[16];
              sm100::tmem_ld<16>(tO + lrow + 16 * hf, o);
              uint32_t ob[16];
#pragma unroll
              for (int i = 0; i < 16; ++i) ob[i] = __float_as_uint(o[i] * al);
              sm100::tmem_st16(tO + lrow + 16 * hf, ob);
            }
          }
        }
#pragma unroll
        for (int i = 0; i < (kKeys - kPoly) / 2; ++i) p[i] = sm100::pack_half2(ex2f(s[2 * i]), ex2f(s[2 * i + 1]));
#pragma unroll
        for (int i = (kKeys - kPoly) / 2; i < kKeys / 2; ++i) p[i] = exp2_poly2(s[2 * i], s[2 * i + 1]);
      } else {
#pragma unroll
        for (int i = 0; i < kKeys / 2; ++i) p[i] = 0u;
      }
      // Qm_b for the QK^T of chunk c+2 (issued after p_ready(c))
      const bool upd = m != mu;
      if (upd) {
        *reinterpret_cast<__half*>(sQm + b * kQBytes + r * 32 + 16 * ((r >> 2) & 1)) = __float2half_rn(-m);
        mu = m;
      }
      if (__any_sync(0xffffffffu, upd)) sm100::fence_proxy_async();
      sm100::tmem_st16(tP + 16 * b + lrow, p);
      sm100::tmem_wait_st();
      sm100::tc_fence_before();
      __syncwarp();
      if (lane == 0) sm100::mbar_arrive(&p_ready[b]);
      if (warp == 2 && lane == 0) ATR(4, c);
    };
    int c = 0;
    for (; c + 1 < nch; c += 2) {
      chunk(c, 0);
      chunk(c + 1, 1);
    }
    if (c < nch) chunk(c, 0);
    // (4) O / l -> fp16
    if (warp == 2 && lane == 0) ATR(0, 3);
    WAIT(&o_full, 0);
    if (warp == 2 && lane == 0) ATR(0, 4);
    sm100::tc_fence_after();
    float o[32];
    sm100::tmem_ld<32>(tO + lrow, o);
    if (valid) {
      const float l = o[16];
      const float inv = l > 0.f ? 1.f / l : 0.f;
      uint32_t pk[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) pk[i] = sm100::pack_half2(o[2 * i] * inv, o[2 * i + 1] * inv);
      uint4* dst = reinterpret_cast<uint4*>(out + (n0 + row) * dmodel + h * kDh);
      dst[0] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
      dst[1] = make_uint4(pk[4], pk[5], pk[6], pk[7]);
    }
  }
  sm100::tc_fence_before();
  __syncthreads();
  if (warp == 1) sm100::tmem_dealloc<128>(tmem);
  if (threadIdx.x == 0) ATR(0, 6);
}

}  // namespace

bool attention_tc_supported(const predtop_dag_s* dag, int d, int H) {
  return d / H == kDh && dag->desc.max_nodes <= 1024;
}

predtop_status attention_tc_launch(const predtop_dag_s* dag, int d, int H, const __half* qkv, __half* out,
                                   cudaStream_t st) {
  const int G = dag->desc.num_graphs;
  const int maxn = dag->desc.max_nodes;
  const int krows_cap = ((maxn + 127) / 128) * 128;
  const int nch_cap = (maxn + kKeys - 1) / kKeys;
  // >= 46 KB: at most 4 CTAs per SM, so the four 128-column TMEM allocations
  // never wait for each other
  const size_t smem = std::max<size_t>(1024 + 3 * kQBytes + 1024 + (size_t)krows_cap * 64 + (size_t)nch_cap * kVtBytes,
                                       46 * 1024);
  PT_SMEM_ATTR(k_attn_tc, smem);
  CUtensorMap tq;
  if (!encode_tma_2d(&tq, qkv, 2, (uint64_t)3 * d, (uint64_t)dag->desc.total_nodes, kDh, 128))
    return PREDTOP_ERR_CUDA;
  const int64_t blocks = std::max<int64_t>(1, dag->qtiles_bound) * H;
  if (blocks > 0x7fffffff) {
    set_error("too many attention work items");
    return PREDTOP_ERR_TOO_LARGE;
  }
  k_attn_tc<<<(unsigned)blocks, kThreads, smem, st>>>(tq, dag->d, G, H, d, qkv, out, krows_cap);
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

}  // namespace predtop

#ifdef PREDTOP_TRACE
extern "C" PREDTOP_API int predtop_debug_attn_trace(unsigned long long* out) {
  return cudaMemcpyFromSymbol(out, predtop::g_at, sizeof(predtop::g_at)) == cudaSuccess ? 0 : -7;
}
#endif
