// attention_tc.cu -- K6 on the 5th-generation tensor cores: reachability-
// masked multi-head attention, Eqn 1, reading R1,
//     O_h = softmax(Q_h K_h^T / sqrt(d_h) + M) V_h,  M(u,v) = 0 iff bit M[u][v]
//     of M = R | R^T | I is set (DAGRA), else -inf.
//
// One CTA = one (graph, 128-row query tile, head); two CTAs per SM (256 TMEM
// columns each), 8 softmax warps per CTA.  Each query row is one TMEM lane;
// the two softmax warps of a lane quarter own the even and the odd 64-key
// chunks, so a softmax thread owns (row, chunk): no shuffles, and the two
// warps sharing a scheduler run half a chunk apart.
//
//   warp 0      TMA producer: the Q tile, then K and V of every 64-key chunk
//               of the graph's head through a kKV-stage ring (SW64 boxes at
//               d_h = 32, SW32 at d_h = 16)
//   warp 1      TMEM owner + MMA issuer (one thread):
//                 S_b  = Q K_c^T + Qm One^T     SS-MMA, M=128 N=64: q.k - m
//                 [O | l] += P_b [V_c | 1]      TS-MMA (A = P in TMEM), N =
//                                               d_h + 16: V is the MN-major B
//                                               operand as TMA wrote it (no
//                                               transpose), a constant ones
//                                               atom LBO bytes after it gives
//                                               the row sums l
//   warps 2..9  softmax: exp2, P as fp16 masked by the bitset and written
//               over its own S_b (tcgen05.st), then O / l -> fp16.
//
// TMEM (256 columns): S_0 | S_1 | S_2 (64 each) | O (d_h) | l (16).  P of
// keys 0-31 of a chunk sits in columns [0,16) of its S, keys 32-63 in
// [32,48) (each 32-key half is read before it is overwritten).  QK^T of chunk c+3 is issued right after PV of chunk c, so the tensor
// core runs two chunks (128 keys) ahead of the softmax.
//
// Softmax in log2 units (Q pre-scaled by log2(e)/sqrt(d_h) in the QKV
// epilogue) against a FIXED per-row reference m = the row's diagonal score
// (allowed: M includes I), rounded to fp16 (it enters the MMA as the fp16
// operand Qm, so the MMA returns s - m).  P = exp2(s - m) is rounded to fp16
// (relative error 2^-11 at any magnitude) while s - m < 16; a row where some
// allowed score exceeds its diagonal by 16 or more (never seen with the
// synthetic models; possible with peaked trained attention) gets P = inf, so
// its row sum l (from the same MMA) is not finite, and it is recomputed
// exactly at the end by its softmax thread on the CUDA cores (fp32 two-pass
// softmax over the row, from the same fp16 q/k/v; rare path).  The check costs
// nothing per chunk.  No per-chunk rescaling, so the two key-half threads of a
// row never need to agree on a moving maximum.
#include <algorithm>

#include "internal.h"
#include "sm100.cuh"
#include "attn_exact.cuh"

namespace predtop {

namespace {

constexpr int kRows = 128;   // query rows per CTA (TMEM lanes)
// Geometry: PREDTOP_ATTN_GEO=64 (default): 64-key chunks, 3 S buffers, 8
// softmax warps (two key halves per row), 256 TMEM columns, 2 CTAs per SM.
// =32: 32-key chunks, 2 S buffers, 4 softmax warps (one thread per row),
// 128 TMEM columns, 4 CTAs per SM.
#ifndef PREDTOP_ATTN_GEO
#define PREDTOP_ATTN_GEO 64
#endif
constexpr int kCh = PREDTOP_ATTN_GEO;          // keys per chunk (S columns)
constexpr int kSBuf = kCh == 64 ? 3 : 2;       // S/P buffers in TMEM
// PREDTOP_ATTN_PAR: 2 (default with 64-key chunks) = each softmax warp owns
// whole chunks of one parity; 3 = twelve softmax warps, one per (lane
// quarter, S buffer) (measured equal to 2); 0 = two warps split every chunk
// into key halves (1-2 % slower on MoE: the two warps of a lane quarter run in
// lockstep on the same S buffer)
#ifndef PREDTOP_ATTN_PAR
#define PREDTOP_ATTN_PAR (PREDTOP_ATTN_GEO == 64 ? 2 : 0)
#endif
constexpr int kPar = PREDTOP_ATTN_PAR;
constexpr int kSoftWarps = kPar == 3 ? 12 : kCh == 64 ? 8 : 4;  // softmax warps (kSoftWarps / 4 threads per row)
constexpr int kTmemCols = kCh == 64 ? 256 : 128;
constexpr int kMinBlocks = kCh == 64 ? 2 : 4;
#ifndef PREDTOP_ATTN_KV
#define PREDTOP_ATTN_KV (kSBuf == 3 ? 5 : 4)
#endif
constexpr int kKV = PREDTOP_ATTN_KV;  // K/V ring stages
static_assert(kKV > kSBuf && kKV <= 2 * kSBuf, "K/V stages are released through s_full (see the producer)");
static_assert(kPar || kCh * 4 / kSoftWarps == 32, "every softmax thread owns 32 keys of a chunk");
static_assert(kPar == 0 || (kCh == 64 && (kPar == 2 || kPar == kSBuf)), "chunk ownership strides");
constexpr int kOutSplit = kCh == 64 ? 2 : 1;  // threads per row writing the output
// PREDTOP_ATTN_SPLIT=1: QK^T and PV are issued by two threads in
// two warps (warp 1 and warp 10), so neither issue stream waits for the
// other's instructions (a tcgen05.mma costs its issuing thread ~75-120 cycles
// next to busy softmax warps); QK^T(c+3) waits for PV(c) through pv_done.
// Measured no faster on MoE (14.1 vs 14.0 ms/step), so off by default.
#ifndef PREDTOP_ATTN_SPLIT
#define PREDTOP_ATTN_SPLIT 0
#endif
constexpr int kSplit = PREDTOP_ATTN_SPLIT;
constexpr int kThreads = 64 + 32 * kSoftWarps + 32 * kSplit;
constexpr int kPvWarp = kSplit ? 2 + kSoftWarps : 1;
// mask words are loaded kMpf chunks ahead of their use
#ifndef PREDTOP_ATTN_MPF
#define PREDTOP_ATTN_MPF 2
#endif
constexpr int kMpf = PREDTOP_ATTN_MPF;


template <int DH>
struct TcCfg {
  static constexpr int RB = DH * 2;        // bytes per Q/K/V row = swizzle width (32 or 64)
  static constexpr int QB = kRows * RB;    // Q tile
  static constexpr int KB = kCh * RB;      // one K (or V) chunk
  static constexpr int STAGE = 3 * KB;     // K | V | ones (the l columns of the PV operand)
  static constexpr int QM = kRows * 32;    // Qm: [128][16] fp16, SW32, column 0 = -m
  static constexpr int ONE = kCh * 32;     // One: [64][16] fp16, SW32, column 0 = 1
  static constexpr int TO = kSBuf * kCh;   // TMEM column of O
  static constexpr int TL = TO + DH;       // TMEM column of l
  static constexpr int BYTES = 1024 + 2 * QB + kKV * STAGE + QM + ONE;
  // > 228/(kMinBlocks+1) KB: at most kMinBlocks CTAs per SM, so the TMEM
  // allocations never wait for each other
  static constexpr int FLOOR = (228 / (kMinBlocks + 1) + 2) * 1024;
  static constexpr int SMEM = BYTES > FLOOR ? BYTES : FLOOR;
  static_assert(TL + 16 <= kTmemCols, "TMEM budget");
};

#ifdef PREDTOP_ATTN_MMA_SPIN
#define MMA_WAIT sm100::mbar_wait
#else
#define MMA_WAIT sm100::mbar_wait_sleep
#endif

#ifdef PREDTOP_TRACE
// debug timeline of one CTA (clock64 at pipeline events, tools/attn_trace.py)
__device__ unsigned long long g_at[8][64];
#define ATR(k, i) \
  do {            \
    if (blockIdx.x == 3001 && (i) < 64) g_at[k][i] = clock64(); \
  } while (0)
#else
#define ATR(k, i) \
  do {            \
  } while (0)
#endif

__device__ __forceinline__ float ex2f(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

// mbarrier helpers on precomputed shared-space addresses (the chunk loop does
// not re-derive them)
__device__ __forceinline__ void bar_wait(uint32_t addr, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@!P1 bra WAIT_%=;\n}" ::"r"(addr),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bar_arrive(uint32_t addr) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(addr) : "memory");
}

template <int DH>
__global__ void __launch_bounds__(kThreads, kMinBlocks)
    k_attn_tc(const __grid_constant__ CUtensorMap tq, const __grid_constant__ CUtensorMap tm, DagDev d, int G,
              int H, int dmodel, const __half* __restrict__ qkv, __half* __restrict__ out, int nmin) {
  using C = TcCfg<DH>;
  extern __shared__ unsigned char dsm[];
  unsigned char* base = sm100::align1024(dsm);
  unsigned char* sQ = base;                      // [128][DH], swizzled
  unsigned char* sKd = sQ + C::QB;               // the tile's own K rows (diagonal scores)
  unsigned char* sKV = sKd + C::QB;              // stage s: K at s*STAGE, V at +KB, ones at +2KB
  unsigned char* sQm = sKV + kKV * C::STAGE;
  unsigned char* sOne = sQm + C::QM;
  __shared__ __align__(8) uint64_t q_full, init_done, kv_full[kKV], s_full[kSBuf],
      p_ready[kSBuf], pv_done[kSBuf], o_full;
  __shared__ uint32_t tmem_slot;

  const int h = blockIdx.x % H;
  const int widx = blockIdx.x / H;
  if (widx >= d.qtile_off[G]) return;
  const int2 wk = d.work[widx];
  const int g = wk.x, qt = wk.y;
  if ((unsigned)g >= (unsigned)G) return;
  const int64_t n0 = d.node_ptr[g];
  const int N = (int)(d.node_ptr[g + 1] - n0);
  if (N < nmin) return;  // a smaller graph: the mma.sync kernel's (attention.cu)
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
  if (threadIdx.x == 0) ATR(2, 0);  // CTA start

  if (threadIdx.x == 0) {
    sm100::mbar_init(&q_full, 1);
    sm100::mbar_init(&init_done, 1);
#pragma unroll
    for (int s = 0; s < kKV; ++s) {
      sm100::mbar_init(&kv_full[s], 1);
    }
#pragma unroll
    for (int b = 0; b < kSBuf; ++b) {
      sm100::mbar_init(&s_full[b], 1);
      sm100::mbar_init(&p_ready[b], kPar ? 4 : kSoftWarps);
      sm100::mbar_init(&pv_done[b], 1);
    }
    sm100::mbar_init(&o_full, 1);
    sm100::fence_mbar_init();
  }
  if (warp == 1) sm100::tmem_alloc<kTmemCols>(&tmem_slot);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem = tmem_slot;
  if (threadIdx.x == 0) ATR(2, 1);  // barriers + TMEM ready

  if (warp == 0) {
    if (lane == 0) {  // -------------------------------------------- TMA
      sm100::mbar_arrive_expect_tx(&q_full, (uint32_t)(2 * C::QB));
      sm100::tma_load_2d(sQ, &tq, &q_full, h * DH, (int)(n0 + qt * kRows));
      sm100::tma_load_2d(sKd, &tq, &q_full, dmodel + h * DH, (int)(n0 + qt * kRows));
      // stage of chunk c - kKV is free once PV(c - kKV) completed, which the
      // commit of QK(c - kKV + kSBuf) (issued after it) implies: no separate
      // "empty" barrier.  kKV <= 2 kSBuf keeps the parity unambiguous (the
      // next phase of that s_full needs the chunk loaded here).
      int s = 0;
      for (int c = 0; c < nch; ++c) {
        if (c >= kKV) {
          // a parity wait is only unambiguous once the barrier has reached
          // the phase before: the first time round, QK(0..kSBuf-1) first
          if (c == kKV)
            for (int i = 0; i < kSBuf; ++i) sm100::mbar_wait_sleep(&s_full[i], 0u);
          const int j = c - kKV + kSBuf;  // QK(j) commit => PV(c - kKV) done
          sm100::mbar_wait_sleep(&s_full[j % kSBuf], (uint32_t)(j / kSBuf) & 1u);
        }
        unsigned char* st = sKV + s * C::STAGE;
        sm100::mbar_arrive_expect_tx(&kv_full[s], (uint32_t)(2 * C::KB));  // K and V (not the ones)
        sm100::tma_load_2d(st, &tm, &kv_full[s], dmodel + h * DH, (int)(n0 + c * kCh));
        sm100::tma_load_2d(st + C::KB, &tm, &kv_full[s], 2 * dmodel + h * DH, (int)(n0 + c * kCh));
        if (++s == kKV) s = 0;
      }
    }
  } else if (warp == 1 || warp == kPvWarp) {
    if (lane == 0) {  // -------------------------------------------- MMA issuer(s)
      constexpr uint32_t id_qk = sm100::make_idesc_f16(128, kCh);
      constexpr uint32_t id_pv = sm100::make_idesc_f16(128, DH + 16) | (1u << 16);  // B [V|1] MN-major
      // descriptors precomputed once; a byte offset o advances the start
      // address field by o >> 4 (shared addresses < 256 KB: no carry out)
      const uint32_t aKV = sm100::smem_u32(sKV);
      const uint64_t dQ = sm100::make_sdesc<C::RB>(sm100::smem_u32(sQ));
      const uint64_t dK = sm100::make_sdesc<C::RB>(aKV);
      const uint64_t dV = sm100::make_sdesc_lbo<C::RB>(aKV + C::KB, C::KB);
      const uint64_t dQm = sm100::make_sdesc<32>(sm100::smem_u32(sQm));
      const uint64_t dOne = sm100::make_sdesc<32>(sm100::smem_u32(sOne));
      const uint32_t sfull0 = sm100::smem_u32(&s_full[0]), kvfull0 = sm100::smem_u32(&kv_full[0]);
      const uint32_t pvdone0 = sm100::smem_u32(&pv_done[0]);
      int qs = 0, qb = 0;  // stage / S buffer of the next QK^T
      uint32_t qph = 0;    // kv_full parity of stage qs (flips per ring pass)
      auto qk = [&](int c) {
        bar_wait(kvfull0 + 8 * qs, qph);
        ATR(3, c);
        sm100::tc_fence_after();
        const uint32_t tS = tmem + kCh * qb;
        const uint64_t off = (uint64_t)((qs * C::STAGE) >> 4);
#pragma unroll
        for (int ks = 0; ks < DH / 16; ++ks)
          sm100::mma_f16_ss(tS, dQ + 2 * ks, dK + off + 2 * ks, id_qk, ks > 0 ? 1u : 0u);
        sm100::mma_f16_ss(tS, dQm, dOne, id_qk, 1u);
        ATR(4, c);
        sm100::mma_commit_addr(sfull0 + 8 * qb);
        ATR(5, c);
        if (++qs == kKV) {
          qs = 0;
          qph ^= 1u;
        }
        if (++qb == kSBuf) qb = 0;
      };
      auto pv = [&](int c, int s, int b) {
        const uint32_t tP = tmem + kCh * b;
        const uint64_t off = (uint64_t)((s * C::STAGE) >> 4);
#pragma unroll
        for (int kk = 0; kk < kCh / 16; ++kk) {
          const uint32_t acc = (c > 0 || kk > 0) ? 1u : 0u;
          // 16 keys = two 8-row core groups of the MN-major V tile; P of keys
          // 16kk.. at column 8kk (first key half) or 32 + 8(kk-2) (second)
          const uint32_t tA = tP + (kk < 2 ? 8 * kk : 32 + 8 * (kk - 2));
          sm100::mma_f16_ts(tmem + C::TO, tA, dV + off + (uint64_t)((kk * 16 * C::RB) >> 4), id_pv, acc);
        }
      };
      if (warp == 1) {  // QK^T issuer (and, unsplit, PV too)
        sm100::mbar_wait_sleep(&q_full, 0);
        sm100::mbar_wait_sleep(&init_done, 0);
        sm100::tc_fence_after();
        for (int c = 0; c < nch && c < kSBuf; ++c) qk(c);
        int s = 0, b = 0;
        uint32_t pph = 0;
        for (int c = 0; c < nch; ++c) {
          if (kSplit) {
            // S_b is rewritten by QK^T(c+3) once PV(c) has read P_b
            if (c + kSBuf < nch) {
              MMA_WAIT(&pv_done[b], pph);
              sm100::tc_fence_after();
              qk(c + kSBuf);
            }
          } else {
            MMA_WAIT(&p_ready[b], pph);
            ATR(0, c);
            sm100::tc_fence_after();
            pv(c, s, b);
            ATR(1, c);
            if (c + kSBuf < nch) qk(c + kSBuf);
          }
          if (++s == kKV) s = 0;
          if (++b == kSBuf) {
            b = 0;
            pph ^= 1u;
          }
        }
        if (!kSplit) sm100::mma_commit(&o_full);
      } else {  // PV issuer
        int s = 0, b = 0;
        uint32_t pph = 0;
        for (int c = 0; c < nch; ++c) {
          MMA_WAIT(&p_ready[b], pph);
          ATR(0, c);
          sm100::tc_fence_after();
          pv(c, s, b);
          ATR(1, c);
          sm100::mma_commit_addr(pvdone0 + 8 * b);
          if (++s == kKV) s = 0;
          if (++b == kSBuf) {
            b = 0;
            pph ^= 1u;
          }
        }
        sm100::mma_commit(&o_full);
      }
    }
  } else {
    // ---------------------------------------------------------- softmax
    const int t = threadIdx.x - 64;        // 0..255
    const int hf = t >> 7;                 // key half of every chunk
    const int q4 = warp & 3;               // TMEM lane quarter this warp may access
    const int r = 32 * q4 + lane;
    const int row = qt * kRows + r;
    const bool valid = row < N;
    const bool warp_dead = qt * kRows + 32 * q4 >= N;
    const uint32_t lrow = (uint32_t)(32 * q4) << 16;
    const uint64_t* Mrow = d.M + d.row_off[g] + (int64_t)(valid ? row : 0) * W;
    // (1) reference m = the diagonal score q_row . k_row (fp32 from the fp16
    // operands), rounded to fp16: it enters the QK^T MMA as the fp16 Qm entry
    if (hf == 0) {
      // from the TMA'd Q tile and the tile's own K rows (swizzled rows of
      // RB bytes: 16-byte chunk j of row x at x*RB + 16*(j ^ swizzle(x)))
      float m = 0.f;
      sm100::mbar_wait(&q_full, 0);
      if (valid) {
#pragma unroll
        for (int j = 0; j < DH / 8; ++j) {
          const int jj = C::RB == 64 ? (j ^ ((r >> 1) & 3)) : (j ^ ((r >> 2) & 1));
          const uint4 a = *reinterpret_cast<const uint4*>(sQ + r * C::RB + 16 * jj);
          const uint4 bq = *reinterpret_cast<const uint4*>(sKd + r * C::RB + 16 * jj);
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
      // Qm = [-m 0 ... 0] (SW32 K-major: 16-byte chunk j of row x sits at
      // x*32 + 16*(j ^ ((x >> 2) & 1)))
      const uint32_t nm = (uint32_t)__half_as_ushort(__float2half_rn(-m));
      unsigned char* qrow = sQm + r * 32;
      *reinterpret_cast<uint4*>(qrow + 16 * ((r >> 2) & 1)) = make_uint4(nm, 0u, 0u, 0u);
      *reinterpret_cast<uint4*>(qrow + 16 - 16 * ((r >> 2) & 1)) = make_uint4(0u, 0u, 0u, 0u);
    }
    for (int k = t; k < kCh; k += 32 * kSoftWarps) {  // One = [1 0 ... 0] per key
      const int o0 = 16 * ((k >> 2) & 1);
      *reinterpret_cast<uint4*>(sOne + k * 32 + o0) = make_uint4(0x3C00u, 0u, 0u, 0u);
      *reinterpret_cast<uint4*>(sOne + k * 32 + 16 - o0) = make_uint4(0u, 0u, 0u, 0u);
    }
    // the ones atom of every K/V stage (constant; the TMA never writes it)
    for (int i = t; i < kKV * (C::KB / 16); i += 32 * kSoftWarps) {
      *reinterpret_cast<uint4*>(sKV + (i / (C::KB / 16)) * C::STAGE + 2 * C::KB + (i % (C::KB / 16)) * 16) =
          make_uint4(0x3C003C00u, 0x3C003C00u, 0x3C003C00u, 0x3C003C00u);
    }
    sm100::fence_proxy_async();
    sm100::named_bar<32 * kSoftWarps>(1);
    if (t == 0) sm100::mbar_arrive(&init_done);
    if (t == 0) ATR(2, 2);  // m, Qm, One written
    // (2) chunks.  The 64-bit mask word c covers chunk c; this thread's 32
    // keys are the low (hf = 0) or high (hf = 1) byte of each 16-bit field of
    // the stored layout (internal.h mask_pos: mask_pos(k + 32) = mask_pos(k) + 8).
    const uint32_t sfull0 = sm100::smem_u32(&s_full[0]), pready0 = sm100::smem_u32(&p_ready[0]);
    // P of one 32-key half: exponentials, fp16 pairs, mask (w: this half's
    // four mask bytes in the low byte of every 16-bit field)
    auto half = [&](uint32_t tS, uint64_t w) {
      if (__any_sync(0xffffffffu, w != 0ull)) {
        float s[32];
        uint32_t p[16];
        sm100::tmem_ld<32>(tS, s);
        // the four mask bytes of this key half in one register: byte f
        // holds keys k with (k >> 1) & 3 == f at bit 2 (k >> 3) + (k & 1),
        // so the pair (2i, 2i+1) sits at bits 8f + 2q, +1 (f = i & 3,
        // q = i >> 2).  The mask is applied after the exponential, to the
        // packed fp16 pair: x0[q] / x1[q] move bit 2q / 2q+1 of every byte to
        // the byte's sign bit, and one sign-replicating byte permute per pair
        // builds its 0xFFFF / 0x0000 halves (a masked score's exponential,
        // inf included, is ANDed away)
        const uint32_t w32 = __byte_perm((uint32_t)w, (uint32_t)(w >> 32), 0x6420);
        uint32_t x0[4], x1[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          x0[q] = w32 << (7 - 2 * q);
          x1[q] = w32 << (6 - 2 * q);
        }
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          const int f = i & 3, q = i >> 2;
          // selector nibbles (result bytes 0..3): x0 byte f, x0 byte f,
          // x1 byte f, x1 byte f, each with the sign-replicate bit 8
          const uint32_t sel = 0xCC88u + 0x1111u * (uint32_t)f;
          uint32_t m;
          asm("prmt.b32 %0, %1, %2, %3;" : "=r"(m) : "r"(x0[q]), "r"(x1[q]), "r"(sel));
          p[i] = sm100::pack_half2(ex2f(s[2 * i]), ex2f(s[2 * i + 1])) & m;
        }
        sm100::tmem_st16(tS, p);
      } else {
        sm100::tmem_st16_zero(tS);
      }
    };
#ifdef PREDTOP_ATTN_MASK_ONES
    constexpr uint64_t kOnes = 0x00FF00FF00FF00FFull;  // timing diagnostic only: every pair allowed
#endif
#if PREDTOP_ATTN_PAR
    // chunk ownership: warp (q4, hf) owns ALL 64 keys of the chunks c with
    // c % kPar == hf, so the warps of a lane quarter run staggered instead of
    // in lockstep on the same S buffer
    const uint32_t tR = tmem + lrow;
    uint64_t wq[kMpf];
#pragma unroll
    for (int i = 0; i < kMpf; ++i) wq[i] = (valid && hf + kPar * i < nch) ? __ldg(Mrow + hf + kPar * i) : 0ull;
#pragma unroll 1
    for (int c = hf; c < nch; c += kPar) {
      const int b = c % kSBuf;
      const uint32_t ph = (uint32_t)(c / kSBuf) & 1u;
#ifdef PREDTOP_ATTN_MASK_ONES
      const uint64_t w = kOnes;
#else
      const uint64_t w = wq[0];
#endif
#pragma unroll
      for (int i = 0; i + 1 < kMpf; ++i) wq[i] = wq[i + 1];
      if (c + kPar * kMpf < nch && valid) wq[kMpf - 1] = __ldg(Mrow + c + kPar * kMpf);
      bar_wait(sfull0 + 8 * b, ph);
      if (lane == 0 && warp == 2) ATR(6, c);
      sm100::tc_fence_after();
      if (!warp_dead) {
        half(tR + kCh * b, w & 0x00FF00FF00FF00FFull);
        half(tR + kCh * b + 32, (w >> 8) & 0x00FF00FF00FF00FFull);
        sm100::tmem_wait_st();
        sm100::tc_fence_before();
      }
      __syncwarp();
      if (lane == 0) bar_arrive(pready0 + 8 * b);
      if (lane == 0 && warp == 2) ATR(7, c);
    }
#else
    const uint32_t tS0 = tmem + 32 * hf + lrow;
    // mask words two chunks ahead (L2 latency).  This thread's 32 keys of
    // chunk c start at key kCh c + 32 hf: word (kCh c + 32 hf) >> 6, byte
    // half ((kCh c + 32 hf) >> 5) & 1 of every 16-bit field.
    auto word_of = [&](int c) -> int { return (kCh * c + 32 * hf) >> 6; };
    uint64_t wq[kMpf];
#pragma unroll
    for (int i = 0; i < kMpf; ++i) wq[i] = (valid && i < nch) ? __ldg(Mrow + word_of(i)) : 0ull;
    int b = 0;
    uint32_t ph = 0;  // phase parity of buffer b's barriers
#pragma unroll 1
    for (int c = 0; c < nch; ++c) {
#ifdef PREDTOP_ATTN_MASK_ONES
      const uint64_t w = kOnes;
#else
      const uint64_t w = (wq[0] >> (8 * (((kCh * c + 32 * hf) >> 5) & 1))) & 0x00FF00FF00FF00FFull;
#endif
#pragma unroll
      for (int i = 0; i + 1 < kMpf; ++i) wq[i] = wq[i + 1];
      if (c + kMpf < nch && valid) wq[kMpf - 1] = __ldg(Mrow + word_of(c + kMpf));
      bar_wait(sfull0 + 8 * b, ph);
      if (lane == 0 && warp == 2) ATR(6, c);
      sm100::tc_fence_after();
      if (!warp_dead) {
        half(tS0 + kCh * b, w);
        sm100::tmem_wait_st();
        sm100::tc_fence_before();
      }
      __syncwarp();
      if (lane == 0) bar_arrive(pready0 + 8 * b);
      if (lane == 0 && warp == 2) ATR(7, c);
      if (++b == kSBuf) {
        b = 0;
        ph ^= 1u;
      }
    }
#endif
    // (3) O / l -> fp16: threads hf < kOutSplit write output columns
    // [OC hf, OC (hf+1)), OC = DH / kOutSplit
    if (t == 0) ATR(2, 3);  // softmax done
    sm100::mbar_wait(&o_full, 0);
    sm100::tc_fence_after();
    if (t == 0) ATR(2, 4);  // O complete
    float o[DH];
    sm100::tmem_ld<DH>(tmem + C::TO + lrow, o);
    float lv[16];
    sm100::tmem_ld<16>(tmem + C::TL + lrow, lv);
    if (valid && hf < kOutSplit) {
      __half* orow = out + (n0 + row) * dmodel + h * DH;
      // a P that overflowed fp16 (s - m >= 16: inf) or a NaN score leaves l
      // non-finite; both key-half threads read the same l, so they agree
      if (!(fabsf(lv[0]) <= 3.0e38f)) {
        if (hf == 0) exact_row<DH>(qkv, n0, N, row, h, dmodel, Mrow, orow);
      } else {
        const float inv = lv[0] > 0.f ? 1.f / lv[0] : 0.f;
        constexpr int OC = DH / kOutSplit;
        uint32_t pk[OC / 2];
#pragma unroll
        for (int i = 0; i < OC / 2; ++i) {
          const float a0 = hf ? o[OC + 2 * i] : o[2 * i];
          const float a1 = hf ? o[OC + 2 * i + 1] : o[2 * i + 1];
          pk[i] = sm100::pack_half2(a0 * inv, a1 * inv);
        }
        uint4* dst = reinterpret_cast<uint4*>(orow + OC * hf);
#pragma unroll
        for (int j = 0; j < OC / 8; ++j) dst[j] = make_uint4(pk[4 * j], pk[4 * j + 1], pk[4 * j + 2], pk[4 * j + 3]);
      }
    }
  }
  sm100::tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0) ATR(2, 5);  // all stored
  if (warp == 1) sm100::tmem_dealloc<kTmemCols>(tmem);
}

template <int DH>
predtop_status launch_tc(const predtop_dag_s* dag, int d, int H, const __half* qkv, __half* out, cudaStream_t st,
                         unsigned blocks, int nmin) {
  using C = TcCfg<DH>;
  PT_SMEM_ATTR(k_attn_tc<DH>, C::SMEM);
  CUtensorMap tq, tm;
  if (!encode_tma_2d(&tq, qkv, 2, (uint64_t)3 * d, (uint64_t)dag->desc.total_nodes, DH, kRows) ||
      !encode_tma_2d(&tm, qkv, 2, (uint64_t)3 * d, (uint64_t)dag->desc.total_nodes, DH, kCh))
    return PREDTOP_ERR_CUDA;
  k_attn_tc<DH><<<blocks, kThreads, C::SMEM, st>>>(tq, tm, dag->d, dag->desc.num_graphs, H, d, qkv, out, nmin);
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

}  // namespace

bool attention_tc_supported(const predtop_dag_s* dag, int d, int H) {
  (void)dag;
  return d / H == 16 || d / H == 32;
}

predtop_status attention_tc_launch(const predtop_dag_s* dag, int d, int H, const __half* qkv, __half* out,
                                   cudaStream_t st, int nmin) {
  const int64_t blocks = std::max<int64_t>(1, dag->qtiles_bound) * H;
  if (blocks > 0x7fffffff) {
    set_error("too many attention work items");
    return PREDTOP_ERR_TOO_LARGE;
  }
  if (d / H == 32) return launch_tc<32>(dag, d, H, qkv, out, st, (unsigned)blocks, nmin);
  if (d / H == 16) return launch_tc<16>(dag, d, H, qkv, out, st, (unsigned)blocks, nmin);
  set_error("unsupported head dim %d", d / H);
  return PREDTOP_ERR_UNSUPPORTED;
}

}  // namespace predtop

#ifdef PREDTOP_TRACE
extern "C" PREDTOP_API int predtop_debug_attn_trace(unsigned long long* out) {
  return cudaMemcpyFromSymbol(out, predtop::g_at, sizeof(predtop::g_at)) == cudaSuccess ? 0 : -7;
}
#endif
