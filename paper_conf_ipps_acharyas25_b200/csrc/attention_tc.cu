// attention_tc.cu -- K6 on the 5th-generation tensor cores: reachability-
// masked multi-head attention, Eqn 1, reading R1,
//     O_h = softmax(Q_h K_h^T / sqrt(d_h) + M) V_h,  M(u,v) = 0 iff bit M[u][v]
//     of M = R | R^T | I is set (DAGRA), else -inf.
//
// One CTA = one (graph, 128-row query tile, head); four CTAs per SM (128 TMEM
// columns each, 16 softmax warps per SM to hide the TMEM/MUFU latencies).
// Every query row is one TMEM lane, so a softmax thread owns a whole row: no
// shuffles, 32 independent exponentials per key chunk.
//
//   warp 0      TMA producer: the Q tile, then K and V of every 32-key chunk
//               of the graph's head through a kKV-stage ring (SW64 boxes at
//               d_h = 32, SW32 at d_h = 16)
//   warp 1      TMEM owner + MMA issuer (one thread):
//                 S_b  = Q K_c^T + Qm_b One^T   SS-MMA, M=128 N=32: q.k - m
//                 O   += P_b V_c                TS-MMA (A = P in TMEM), V is
//                                               the MN-major B operand as TMA
//                                               wrote it (no transpose)
//   warps 2..5  softmax (row = TMEM lane): mask bits -> -inf, exp2, P as fp16
//               written over S_b (tcgen05.st), row sums l in registers
//               (fp32), then O / l -> fp16 rows.
//
// TMEM (128 columns): S_0 | S_1 | S_2 (32 each, P in the first 16 of its S)
// | O (d_h).  QK^T of chunk c+3 is issued right after PV of chunk c, so the
// tensor core runs two chunks ahead of the softmax.
//
// Online softmax in log2 units (Q pre-scaled by log2(e)/sqrt(d_h) in the QKV
// epilogue).  The reference m of a row starts at its diagonal score (M
// includes I, so the row max is >= it) and only moves when some P of a chunk
// exceeds 2^12 (or overflows fp16): then m moves to the chunk max (fp16-
// rounded; it enters the MMA as the fp16 operand Qm) and O, l are rescaled in
// TMEM once the previous PV has completed (rare).  S_b was computed with the
// m held in Qm_b when its QK^T was issued (mu_b); a row whose m moved since
// corrects by m - mu_b.
#include <algorithm>

#include "internal.h"
#include "sm100.cuh"

namespace predtop {

namespace {

constexpr int kRows = 128;   // query rows per CTA (TMEM lanes)
constexpr int kCh = 32;      // keys per chunk (S columns)
constexpr int kSBuf = 3;     // S/P buffers in TMEM
constexpr int kKV = 8;       // K/V ring stages
constexpr int kThreads = 192;
constexpr float kPMax = 4096.f;  // P above this (or inf) moves the reference m

template <int DH>
struct TcCfg {
  static constexpr int RB = DH * 2;        // bytes per Q/K/V row = swizzle width (32 or 64)
  static constexpr int QB = kRows * RB;    // Q tile
  static constexpr int KB = kCh * RB;      // one K (or V) chunk
  static constexpr int STAGE = 2 * KB;     // K | V
  static constexpr int QM = kRows * 32;    // Qm_b: [128][16] fp16, SW32, column 0 = -m
  static constexpr int ONE = kCh * 32;     // One: [32][16] fp16, SW32, column 0 = 1
  static constexpr int TO = kSBuf * kCh;   // TMEM column of O
  static constexpr int BYTES = 1024 + QB + kKV * STAGE + kSBuf * QM + ONE;
  // > 228/5 KB: at most four CTAs per SM, so the 128-column TMEM
  // allocations never wait for each other
  static constexpr int SMEM = BYTES > 47 * 1024 ? BYTES : 47 * 1024;
  static_assert(TO + DH <= 128, "TMEM budget");
};

#ifdef PREDTOP_ATTN_MMA_SPIN
#define MMA_WAIT sm100::mbar_wait
#else
#define MMA_WAIT sm100::mbar_wait_sleep
#endif

__device__ __forceinline__ float ex2f(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

// bit of key k (0..63 of a 64-key mask word) in the stored layout
// (internal.h mask_pos)
__device__ __forceinline__ bool key_bit(uint32_t lo, uint32_t hi, int k) {
  const int p = mask_pos(k);
  return p < 32 ? ((lo >> p) & 1u) : ((hi >> (p - 32)) & 1u);
}

template <int DH>
__global__ void __launch_bounds__(kThreads, 4)
    k_attn_tc(const __grid_constant__ CUtensorMap tq, const __grid_constant__ CUtensorMap tm, DagDev d, int G, int H, int dmodel,
              const __half* __restrict__ qkv, __half* __restrict__ out) {
  using C = TcCfg<DH>;
  extern __shared__ unsigned char dsm[];
  unsigned char* base = sm100::align1024(dsm);
  unsigned char* sQ = base;                      // [128][DH], swizzled
  unsigned char* sKV = sQ + C::QB;               // stage s: K at s*STAGE, V at +KB
  unsigned char* sQm = sKV + kKV * C::STAGE;     // Qm_b at b*QM
  unsigned char* sOne = sQm + kSBuf * C::QM;
  __shared__ __align__(8) uint64_t q_full, init_done, kv_full[kKV], kv_empty[kKV], s_full[kSBuf],
      p_ready[kSBuf], pv_done[2], o_full;
  __shared__ uint32_t tmem_slot;

  const int h = blockIdx.x % H;
  const int widx = blockIdx.x / H;
  if (widx >= d.qtile_off[G]) return;
  const int2 wk = d.work[widx];
  const int g = wk.x, qt = wk.y;
  if ((unsigned)g >= (unsigned)G) return;
  const int64_t n0 = d.node_ptr[g];
  const int N = (int)(d.node_ptr[g + 1] - n0);
  if (d.status[g] != PREDTOP_OK) {
    // an invalid graph (latency NaN) still gets finite zero rows, so no NaN
    // reaches a neighbouring graph's K/V chunk in the next layer
    for (int i = threadIdx.x; i < kRows * (DH / 8); i += kThreads) {
      const int row = qt * kRows + i / (DH / 8);
      if (row < N)
        *reinterpret_cast<uint4*>(out + (n0 + row) * dmodel + h * DH + 8 * (i % (DH / 8))) = make_uint4(0, 0, 0, 0);
    }
    return;
  }
  const int W = 2 * ((N + 127) / 128);
  const int nch = (N + kCh - 1) / kCh;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    sm100::mbar_init(&q_full, 1);
    sm100::mbar_init(&init_done, 1);
#pragma unroll
    for (int s = 0; s < kKV; ++s) {
      sm100::mbar_init(&kv_full[s], 1);
      sm100::mbar_init(&kv_empty[s], 1);
    }
#pragma unroll
    for (int b = 0; b < kSBuf; ++b) {
      sm100::mbar_init(&s_full[b], 1);
      sm100::mbar_init(&p_ready[b], 4);
    }
    sm100::mbar_init(&pv_done[0], 1);
    sm100::mbar_init(&pv_done[1], 1);
    sm100::mbar_init(&o_full, 1);
    sm100::fence_mbar_init();
  }
  if (warp == 1) sm100::tmem_alloc<128>(&tmem_slot);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem = tmem_slot;

  if (warp == 0) {
    if (lane == 0) {  // -------------------------------------------- TMA
      const int r0 = (int)(n0 + qt * kRows);
      sm100::mbar_arrive_expect_tx(&q_full, (uint32_t)C::QB);
      sm100::tma_load_2d(sQ, &tq, &q_full, h * DH, r0);
      for (int c = 0; c < nch; ++c) {
        const int s = c % kKV;
        if (c >= kKV) sm100::mbar_wait_sleep(&kv_empty[s], ((c / kKV) - 1) & 1);
        unsigned char* st = sKV + s * C::STAGE;
        sm100::mbar_arrive_expect_tx(&kv_full[s], (uint32_t)C::STAGE);
        sm100::tma_load_2d(st, &tm, &kv_full[s], dmodel + h * DH, (int)(n0 + c * kCh));
        sm100::tma_load_2d(st + C::KB, &tm, &kv_full[s], 2 * dmodel + h * DH, (int)(n0 + c * kCh));
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {  // -------------------------------------------- MMA issuer
      constexpr uint32_t id_qk = sm100::make_idesc_f16(128, kCh);
      constexpr uint32_t id_pv = sm100::make_idesc_f16(128, DH) | (1u << 16);  // B (V) MN-major
      const uint32_t aQ = sm100::smem_u32(sQ), aKV = sm100::smem_u32(sKV);
      const uint32_t aQm = sm100::smem_u32(sQm), aOne = sm100::smem_u32(sOne);
      auto qk = [&](int c) {
        const int s = c % kKV, b = c % kSBuf;
        sm100::mbar_wait_sleep(&kv_full[s], (c / kKV) & 1);
        sm100::tc_fence_after();
        const uint32_t tS = tmem + kCh * b;
#pragma unroll
        for (int ks = 0; ks < DH / 16; ++ks)
          sm100::mma_f16_ss(tS, sm100::make_sdesc<C::RB>(aQ + 32 * ks),
                            sm100::make_sdesc<C::RB>(aKV + s * C::STAGE + 32 * ks), id_qk, ks > 0 ? 1u : 0u);
        sm100::mma_f16_ss(tS, sm100::make_sdesc<32>(aQm + b * C::QM), sm100::make_sdesc<32>(aOne), id_qk, 1u);
        sm100::mma_commit(&s_full[b]);
      };
      sm100::mbar_wait_sleep(&q_full, 0);
      sm100::mbar_wait_sleep(&init_done, 0);
      sm100::tc_fence_after();
      for (int c = 0; c < nch && c < kSBuf; ++c) qk(c);
      for (int c = 0; c < nch; ++c) {
        const int s = c % kKV, b = c % kSBuf;
        MMA_WAIT(&p_ready[b], (c / kSBuf) & 1);
        sm100::tc_fence_after();
        const uint32_t tP = tmem + kCh * b;
        const uint32_t aV = aKV + s * C::STAGE + C::KB;
#pragma unroll
        for (int kk = 0; kk < kCh / 16; ++kk) {
          const uint32_t acc = (c > 0 || kk > 0) ? 1u : 0u;
          // 16 keys = two 8-row core groups of the MN-major V tile
          sm100::mma_f16_ts(tmem + C::TO, tP + 8 * kk, sm100::make_sdesc<C::RB>(aV + kk * 16 * C::RB), id_pv, acc);
        }
        sm100::mma_commit(&kv_empty[s]);
        sm100::mma_commit(&pv_done[c & 1]);
        if (c + kSBuf < nch) qk(c + kSBuf);
      }
      sm100::mma_commit(&o_full);
    }
  } else {
    // ---------------------------------------------------------- softmax
    const int t = threadIdx.x - 64;  // 0..127
    const int q4 = warp & 3;         // TMEM lane quarter this warp may access
    const int r = 32 * q4 + lane;
    const int row = qt * kRows + r;
    const bool valid = row < N;
    const bool warp_dead = qt * kRows + 32 * q4 >= N;
    const uint32_t lrow = (uint32_t)(32 * q4) << 16;
    const uint64_t* Mrow = d.M + d.row_off[g] + (int64_t)(valid ? row : 0) * W;
    // one 64-bit mask word covers two chunks: chunk c uses the keys
    // 32(c&1)..32(c&1)+31 of word c>>1, i.e. the low (c even) or high (c odd)
    // byte of each 16-bit field of the stored layout (internal.h mask_pos:
    // mask_pos(k + 32) = mask_pos(k) + 8)
    uint64_t wword = valid ? __ldg(Mrow) : 0ull;
    // (1) reference m = the diagonal score q_row . k_row (fp32 from the fp16
    // operands), rounded to fp16: it enters the QK^T MMA as the fp16 Qm entry
    float m = 0.f;
    if (valid) {
      const uint4* qr = reinterpret_cast<const uint4*>(qkv + (n0 + row) * 3 * dmodel + h * DH);
      const uint4* kr = reinterpret_cast<const uint4*>(qkv + (n0 + row) * 3 * dmodel + dmodel + h * DH);
#pragma unroll
      for (int j = 0; j < DH / 8; ++j) {
        const uint4 a = __ldg(qr + j), bq = __ldg(kr + j);
        const uint32_t aw[4] = {a.x, a.y, a.z, a.w}, bw[4] = {bq.x, bq.y, bq.z, bq.w};
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const float2 x = __half22float2(*reinterpret_cast<const __half2*>(&aw[i]));
          const float2 y = __half22float2(*reinterpret_cast<const __half2*>(&bw[i]));
          m = fmaf(x.x, y.x, m);
          m = fmaf(x.y, y.y, m);
        }
      }
    }
    m = __half2float(__float2half_rn(m));
    // Qm_b = [-m 0 ... 0] (SW32 K-major: 16-byte chunk j of row x sits at
    // x*32 + 16*(j ^ ((x >> 2) & 1))); One = [1 0 ... 0] per key
    const int qm_off = r * 32 + 16 * ((r >> 2) & 1);
    {
      const uint32_t nm = (uint32_t)__half_as_ushort(__float2half_rn(-m));
#pragma unroll
      for (int b = 0; b < kSBuf; ++b) {
        unsigned char* q = sQm + b * C::QM + r * 32;
        *reinterpret_cast<uint4*>(q + 16 * ((r >> 2) & 1)) = make_uint4(nm, 0u, 0u, 0u);
        *reinterpret_cast<uint4*>(q + 16 - 16 * ((r >> 2) & 1)) = make_uint4(0u, 0u, 0u, 0u);
      }
      if (t < kCh) {
        const int o0 = 16 * ((t >> 2) & 1);
        *reinterpret_cast<uint4*>(sOne + t * 32 + o0) = make_uint4(0x3C00u, 0u, 0u, 0u);
        *reinterpret_cast<uint4*>(sOne + t * 32 + 16 - o0) = make_uint4(0u, 0u, 0u, 0u);
      }
      sm100::fence_proxy_async();
      sm100::named_bar<128>(1);
      if (t == 0) sm100::mbar_arrive(&init_done);
    }
    // (2) chunks.  S_b = q.k - mu_b, mu_b = the m held in Qm_b when QK^T of
    // S_b was issued (read back from Qm_b: m is fp16, so exact).  l: two
    // fp32 partial sums of the unrounded exponentials.
    float l0 = 0.f, l1 = 0.f;
    int b = 0;
#pragma unroll 1
    for (int c = 0; c < nch; ++c) {
      const uint64_t w = ((c & 1) ? (wword >> 8) : wword) & 0x00FF00FF00FF00FFull;
      if ((c & 1) && 2 * ((c >> 1) + 1) < nch && valid) wword = __ldg(Mrow + (c >> 1) + 1);
      sm100::mbar_wait(&s_full[b], (c / kSBuf) & 1);
      sm100::tc_fence_after();
      if (!warp_dead) {
        const uint32_t tS = tmem + kCh * b + lrow;
        __half* qm = reinterpret_cast<__half*>(sQm + b * C::QM + qm_off);
        uint32_t p[kCh / 2];
        if (__any_sync(0xffffffffu, w != 0ull)) {
          float s[kCh];
          sm100::tmem_ld<kCh>(tS, s);
          const float fix = m + __half2float(*qm);  // m - mu_b
          if (__any_sync(0xffffffffu, fix != 0.f)) {
#pragma unroll
            for (int k = 0; k < kCh; ++k) s[k] -= fix;
          }
          const uint32_t wl = (uint32_t)w, wh = (uint32_t)(w >> 32);
#pragma unroll
          for (int k = 0; k < kCh; ++k) s[k] = key_bit(wl, wh, k) ? s[k] : -INFINITY;
          __half2 mx2 = __float2half2_rn(0.f);
          const float lb0 = l0, lb1 = l1;  // sums before this chunk (rare path)
#pragma unroll
          for (int i = 0; i < kCh / 2; ++i) {
            const float e0 = ex2f(s[2 * i]), e1 = ex2f(s[2 * i + 1]);
            p[i] = sm100::pack_half2(e0, e1);
            if (i & 1) {
              l1 += e0 + e1;
            } else {
              l0 += e0 + e1;
            }
            mx2 = __hmax2(mx2, *reinterpret_cast<const __half2*>(&p[i]));
          }
          const float pm = fmaxf(__low2float(mx2), __high2float(mx2));
          const bool over = !(pm <= kPMax);
          if (__any_sync(0xffffffffu, over)) {
            // rare: move m to the chunk maximum and rescale O (TMEM) and l
            // once PV of chunk c-1 (the last writer of O) has completed.
            // s_full(c) implies PV(c-3) completed, so the pv_done parity is
            // unambiguous.
            float mx = -INFINITY;
#pragma unroll
            for (int k = 0; k < kCh; ++k) mx = fmaxf(mx, s[k]);
            const float mn = over ? __half2float(__float2half_rn(m + mx)) : m;
            const float dl = mn - m;
            m = mn;
#pragma unroll
            for (int k = 0; k < kCh; ++k) s[k] -= dl;
            const float al = ex2f(-dl);
            l0 = lb0 * al;
            l1 = lb1 * al;
            if (c > 0) {
              sm100::mbar_wait(&pv_done[(c - 1) & 1], ((c - 1) >> 1) & 1);
              sm100::tc_fence_after();
#pragma unroll 1
              for (int j = 0; j < DH / 16; ++j) {
                float o[16];
                sm100::tmem_ld<16>(tmem + C::TO + lrow + 16 * j, o);
                uint32_t ob[16];
#pragma unroll
                for (int i = 0; i < 16; ++i) ob[i] = __float_as_uint(o[i] * al);
                sm100::tmem_st16(tmem + C::TO + lrow + 16 * j, ob);
              }
            }
#pragma unroll
            for (int i = 0; i < kCh / 2; ++i) {
              const float e0 = ex2f(s[2 * i]), e1 = ex2f(s[2 * i + 1]);
              p[i] = sm100::pack_half2(e0, e1);
              if (i & 1) {
                l1 += e0 + e1;
              } else {
                l0 += e0 + e1;
              }
            }
            if (m != -__half2float(*qm)) {  // Qm_b for the QK^T of chunk c+3
              *qm = __float2half_rn(-m);
            }
            sm100::fence_proxy_async();
          }
        } else {
#pragma unroll
          for (int i = 0; i < kCh / 2; ++i) p[i] = 0u;
        }
        if (m != -__half2float(*qm)) {  // m moved in an earlier chunk: Qm_b catches up
          *qm = __float2half_rn(-m);
          sm100::fence_proxy_async();
        }
        sm100::tmem_st16(tS, p);
        sm100::tmem_wait_st();
        sm100::tc_fence_before();
      }
      __syncwarp();
      if (lane == 0) sm100::mbar_arrive(&p_ready[b]);
      b = b == kSBuf - 1 ? 0 : b + 1;
    }
    // (3) O / l -> fp16
    sm100::mbar_wait(&o_full, 0);
    sm100::tc_fence_after();
    float o[DH];
    sm100::tmem_ld<DH>(tmem + C::TO + lrow, o);
    if (valid) {
      const float l = l0 + l1;
      const float inv = l > 0.f ? 1.f / l : 0.f;
      uint32_t pk[DH / 2];
#pragma unroll
      for (int i = 0; i < DH / 2; ++i) pk[i] = sm100::pack_half2(o[2 * i] * inv, o[2 * i + 1] * inv);
      uint4* dst = reinterpret_cast<uint4*>(out + (n0 + row) * dmodel + h * DH);
#pragma unroll
      for (int j = 0; j < DH / 8; ++j) dst[j] = make_uint4(pk[4 * j], pk[4 * j + 1], pk[4 * j + 2], pk[4 * j + 3]);
    }
  }
  sm100::tc_fence_before();
  __syncthreads();
  if (warp == 1) sm100::tmem_dealloc<128>(tmem);
}

template <int DH>
predtop_status launch_tc(const predtop_dag_s* dag, int d, int H, const __half* qkv, __half* out, cudaStream_t st,
                         unsigned blocks) {
  using C = TcCfg<DH>;
  PT_SMEM_ATTR(k_attn_tc<DH>, C::SMEM);
  CUtensorMap tq, tm;
  if (!encode_tma_2d(&tq, qkv, 2, (uint64_t)3 * d, (uint64_t)dag->desc.total_nodes, DH, kRows) ||
      !encode_tma_2d(&tm, qkv, 2, (uint64_t)3 * d, (uint64_t)dag->desc.total_nodes, DH, kCh))
    return PREDTOP_ERR_CUDA;
  k_attn_tc<DH><<<blocks, kThreads, C::SMEM, st>>>(tq, tm, dag->d, dag->desc.num_graphs, H, d, qkv, out);
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

}  // namespace

bool attention_tc_supported(const predtop_dag_s* dag, int d, int H) {
  (void)dag;
  return d / H == 16 || d / H == 32;
}

predtop_status attention_tc_launch(const predtop_dag_s* dag, int d, int H, const __half* qkv, __half* out,
                                   cudaStream_t st) {
  const int64_t blocks = std::max<int64_t>(1, dag->qtiles_bound) * H;
  if (blocks > 0x7fffffff) {
    set_error("too many attention work items");
    return PREDTOP_ERR_TOO_LARGE;
  }
  if (d / H == 32) return launch_tc<32>(dag, d, H, qkv, out, st, (unsigned)blocks);
  if (d / H == 16) return launch_tc<16>(dag, d, H, qkv, out, st, (unsigned)blocks);
  set_error("unsupported head dim %d", d / H);
  return PREDTOP_ERR_UNSUPPORTED;
}

}  // namespace predtop
