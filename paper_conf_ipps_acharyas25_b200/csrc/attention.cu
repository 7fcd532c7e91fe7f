// attention.cu -- K6: reachability-masked multi-head attention, Eqn 1
// with V (reading R1):
//     O_h = softmax(Q_h K_h^T / sqrt(d_h) + M) V_h,  M(u,v) = 0 iff the mask
//     bit M[u][v] of  M = R | R^T | I  is set (DAGRA), else -inf.
//
// One CTA = one (graph, 128-row query tile, head); 8 warps x 16 query rows.
// The 1-D grid runs the heads of a q-tile back to back, so the q/k/v rows of
// a graph are fetched from HBM once and re-read by the other heads from L2.
//
// Keys/values live in shared memory in 64-key chunks (one chunk = one 64-bit
// word of every mask row), brought in by TMA ([64 keys x d_h] boxes, one
// elected thread, one mbarrier).  Graphs whose K/V fit (N <= ~1500 at d_h =
// 16) are loaded whole, then every warp runs independently; larger graphs
// stream through a 3-stage ring of 256-key stages (two stages in flight).
//
// Per warp (16 query rows) and 16-key block: QK^T on the m16n8k16 tensor-core
// MMA with the accumulator input C = -m (allowed pair) or -inf (masked), so
// the MMA returns s - m directly; a block with no allowed pair among the
// warp's rows is skipped (flags from k_bflags).  Online softmax in log2 units
// (Q pre-scaled in the QKV epilogue), reference m = the row's diagonal score,
// lazy rescaling; P = exp2(s - m) (MUFU ex2) rounded once to fp16; the row
// sums l come from the tensor core (P x an all-ones B fragment).
//
// At d_h = 16/32 the kernel is bound by the exponentials and the issue slots
// around them, not by the tensor pipe: QK^T and PV are 2*d_h flops per score
// each.  The S accumulator fragment is the P operand fragment, so S and P
// never leave registers; see DESIGN.md "K6".  This kernel serves d_h = 16;
// d_h = 32 runs on the tcgen05/TMEM kernel of attention_tc.cu.
#include "internal.h"
#include "sm100.cuh"

namespace predtop {

namespace {

__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

__device__ __forceinline__ void mma16816(float (&d)[4], const uint32_t (&a)[4], uint32_t b0,
                                         uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

__device__ __forceinline__ void ldsm_x4(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2,
                                        uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2,
                                          uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}

__device__ __forceinline__ float dot_h2(uint32_t a, uint32_t b) {
  const float2 x = __half22float2(*reinterpret_cast<const __half2*>(&a));
  const float2 y = __half22float2(*reinterpret_cast<const __half2*>(&b));
  return x.x * y.x + x.y * y.y;
}
__device__ __forceinline__ uint32_t pack_h2(float a, float b) {
  __half2 h = __floats2half2_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}

// D = A*B + C with an explicit accumulator input (QK^T: C = -m or -inf).
__device__ __forceinline__ void mma16816_c(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1,
                                           const float (&c)[4]) {
  asm volatile(
      "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%10,%11,%12,%13};"
      : "=f"(d[0]), "=f"(d[1]), "=f"(d[2]), "=f"(d[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1), "f"(c[0]), "f"(c[1]), "f"(c[2]),
        "f"(c[3]));
}

constexpr int kChunk = 64;
#ifndef PREDTOP_ATTN_MINB32
#define PREDTOP_ATTN_MINB32 3  // CTAs per SM of the 8-warp d_h = 32 kernels (78 registers)
#endif
constexpr int kStages = 3;  // streaming path: a ring of 3 stages of stage_chunks<DH>() 64-key chunks
// d_h = 16: 4 chunks (256 keys, 48 KB of ring, 4 CTAs/SM); d_h = 32: 2 chunks
// (128 keys, 48 KB, so 3 CTAs/SM fit -- 1xB200 MoE attention 20.9 -> 18.3 ms/step
// against 4 chunks at 2 CTAs/SM)
template <int DH>
constexpr int stage_chunks() { return DH == 32 ? 2 : 4; }

// flag nibble f (bit j = block j fully allowed) -> the thread's mask bits of
// those blocks in rows a (bits 0-15) and b (bits 16-31): nibble j of each half
__constant__ uint32_t c_full_bits[16] = {
    0x00000000u, 0x000F000Fu, 0x00F000F0u, 0x00FF00FFu, 0x0F000F00u, 0x0F0F0F0Fu, 0x0FF00FF0u, 0x0FFF0FFFu,
    0xF000F000u, 0xF00FF00Fu, 0xF0F0F0F0u, 0xF0FFF0FFu, 0xFF00FF00u, 0xFF0FFF0Fu, 0xFFF0FFF0u, 0xFFFFFFFFu};

// K and V chunks sit in shared memory in natural key order, as TMA writes a
// [64 keys x d_h] box with the swizzle of its row size (SWIZZLE_32B for d_h =
// 16, 64B for 32): 16-byte piece p of row r is at r*RB + 16*(p ^ sw(r)),
// sw(r) = ((r*RB) >> 7) & (RB/16 - 1).  The mask words are stored permuted
// (internal.h mask_pos) so that the keys of a thread's accumulator fragment
// (n-tile nt, column 2tq+u: key 8nt + 2tq + u) are the contiguous bits
// [16tq, 16tq+16), bit 2nt+u, and 16-key block j is 0x000F000F000F000F << 4j.
template <int DH>
struct Attn {
  static constexpr int RB = DH * 2;     // row bytes (TMA box row, swizzle span)
  static constexpr int KS = DH / 16;    // k-steps for QK^T
  static constexpr int DN = DH / 8;     // n-tiles of the output
  static constexpr int CHUNK_BYTES = kChunk * RB;  // one K or V chunk
  static constexpr int BLK = 16 * RB;   // bytes of a 16-key block

  uint32_t qa[KS][4];
  float o[DN][4];
  float osum[4];  // P x ones (tensor-core row sums l): [0] row a, [2] row b
  float m_a, m_b;
  uint32_t kl[KS], vl[DN / 2];  // per-lane ldmatrix byte offsets (swizzled)

  __device__ __forceinline__ void init(int lane) {
    const int r8 = lane & 7;
    // K (non-transposed x4): matrices (keys 0-7 | 8-15) x (cols 0-7 | 8-15) of
    // the k-step; V (transposed x4): (keys 0-7 | 8-15) x (cols dn*8.. | +8).
    // Block offsets (16 rows) are multiples of 128 B, so sw(r) depends on
    // the lane only.
    const int rk = ((lane >> 4) & 1) * 8 + r8, rv = ((lane >> 3) & 1) * 8 + r8;
    const int swk = ((rk * RB) >> 7) & (RB / 16 - 1), swv = ((rv * RB) >> 7) & (RB / 16 - 1);
#pragma unroll
    for (int ks = 0; ks < KS; ++ks)
      kl[ks] = (uint32_t)(rk * RB + 16 * ((2 * ks + ((lane >> 3) & 1)) ^ swk));
#pragma unroll
    for (int i = 0; i < DN / 2; ++i)
      vl[i] = (uint32_t)(rv * RB + 16 * ((2 * i + ((lane >> 4) & 1)) ^ swv));
#pragma unroll
    for (int i = 0; i < DN; ++i) o[i][0] = o[i][1] = o[i][2] = o[i][3] = 0.f;
    osum[0] = osum[1] = osum[2] = osum[3] = 0.f;
    m_a = m_b = 0.f;  // set to the diagonal score by the kernel
  }

  // One 64-key chunk for the warp's 16 rows.  kbase/vbase: shared addresses of
  // the chunk's (permuted) K and V rows; mk: this thread's 16 mask bits of
  // row a (bits 0-15) and of row b (bits 16-31); fl: block flags of (warp's
  // 16-row group, chunk) from the DAG build (k_bflags): bit j = block j has an
  // allowed pair, bit 4+j = all pairs allowed.
  //
  // The mask and the running reference m enter through the accumulator input
  // of the QK^T MMA: C = -m (allowed) or -inf (masked), so the MMA returns
  // s - m directly and P = exp2(S) needs no subtraction and no select.
  __device__ __forceinline__ void chunk(uint32_t kbase, uint32_t vbase, uint32_t mk, uint32_t fl) {
    const uint32_t act = fl & 15u;
    if (!act) return;
    // fully allowed blocks (flag bits 4-7): set all of the thread's bits of
    // those blocks -- one select per score either way, no second code path
    mk |= c_full_bits[(fl >> 4) & 15u];
    // two 32-key phases (blocks 2ph, 2ph+1): half the live score registers
#pragma unroll
    for (int ph = 0; ph < 2; ++ph) {
      if (!((act >> (2 * ph)) & 3u)) continue;
      const float nma = -m_a, nmb = -m_b;
      float s[4][4];
      float mx = -INFINITY;  // max of s - m over both rows (overflow check only)
#pragma unroll
      for (int jj = 0; jj < 2; ++jj) {
        const int j = 2 * ph + jj;
        if (!(act & (1u << j))) continue;
        float c[2][4];
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          const int e = 2 * (2 * j + u);
          c[u][0] = ((mk >> e) & 1u) ? nma : -INFINITY;
          c[u][1] = ((mk >> (e + 1)) & 1u) ? nma : -INFINITY;
          c[u][2] = ((mk >> (e + 16)) & 1u) ? nmb : -INFINITY;
          c[u][3] = ((mk >> (e + 17)) & 1u) ? nmb : -INFINITY;
        }
#pragma unroll
        for (int ks = 0; ks < KS; ++ks) {
          uint32_t b0, b1, b2, b3;
          ldsm_x4(kbase + kl[ks] + j * BLK, b0, b1, b2, b3);
          if (ks == 0) {
            mma16816_c(s[2 * jj], qa[ks], b0, b1, c[0]);
            mma16816_c(s[2 * jj + 1], qa[ks], b2, b3, c[1]);
          } else {
            mma16816(s[2 * jj], qa[ks], b0, b1);
            mma16816(s[2 * jj + 1], qa[ks], b2, b3);
          }
        }
        const float* x = s[2 * jj];
        const float* y = s[2 * jj + 1];
        mx = fmaxf(fmaxf(mx, fmaxf(x[0], x[1])), fmaxf(fmaxf(x[2], x[3]), fmaxf(y[0], y[1])));
        mx = fmaxf(mx, fmaxf(y[2], y[3]));
      }
      // Lazy rescaling: m starts at the row's diagonal score (always allowed,
      // M includes I) and only moves when a score exceeds it by more than 8
      // (log2 units), so P = exp2(s - m) <= 256 stays exact in fp16.
      if (__any_sync(0xffffffffu, mx > 8.f)) {
        float ma = -INFINITY, mb = -INFINITY;
#pragma unroll
        for (int jj = 0; jj < 2; ++jj) {
          if (!(act & (1u << (2 * ph + jj)))) continue;
          ma = fmaxf(ma, fmaxf(fmaxf(s[2 * jj][0], s[2 * jj][1]), fmaxf(s[2 * jj + 1][0], s[2 * jj + 1][1])));
          mb = fmaxf(mb, fmaxf(fmaxf(s[2 * jj][2], s[2 * jj][3]), fmaxf(s[2 * jj + 1][2], s[2 * jj + 1][3])));
        }
        ma = fmaxf(ma, __shfl_xor_sync(0xffffffffu, ma, 1));
        ma = fmaxf(ma, __shfl_xor_sync(0xffffffffu, ma, 2));
        mb = fmaxf(mb, __shfl_xor_sync(0xffffffffu, mb, 1));
        mb = fmaxf(mb, __shfl_xor_sync(0xffffffffu, mb, 2));
        const float da = ma > 8.f ? ma : 0.f, db = mb > 8.f ? mb : 0.f;
        const float al_a = ex2(-da), al_b = ex2(-db);
#pragma unroll
        for (int i = 0; i < DN; ++i) {
          o[i][0] *= al_a; o[i][1] *= al_a;
          o[i][2] *= al_b; o[i][3] *= al_b;
        }
        osum[0] *= al_a; osum[1] *= al_a;
        osum[2] *= al_b; osum[3] *= al_b;
        m_a += da;
        m_b += db;
#pragma unroll
        for (int nt = 0; nt < 4; ++nt) {
          s[nt][0] -= da; s[nt][1] -= da;
          s[nt][2] -= db; s[nt][3] -= db;
        }
      }
#pragma unroll
      for (int jj = 0; jj < 2; ++jj) {
        const int j = 2 * ph + jj;
        if (!(act & (1u << j))) continue;
        uint32_t pa[4];
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          const int nt = 2 * jj + u;
          pa[2 * u + 0] = pack_h2(ex2(s[nt][0]), ex2(s[nt][1]));
          pa[2 * u + 1] = pack_h2(ex2(s[nt][2]), ex2(s[nt][3]));
        }
#pragma unroll
        for (int dn = 0; dn < DN; dn += 2) {
          uint32_t b0, b1, b2, b3;
          ldsm_x4_t(vbase + vl[dn / 2] + j * BLK, b0, b1, b2, b3);
          mma16816(o[dn], pa, b0, b1);
          mma16816(o[dn + 1], pa, b2, b3);
        }
        // row sums l: P x (16 x 8 all-ones B operand, constant fragments)
        mma16816(osum, pa, 0x3C003C00u, 0x3C003C00u);
      }
    }
  }

};

// NW warps per CTA: 8 (a whole 128-row q-tile) or 4 (half of one: two CTAs
// per work item, so a short last q-tile idles at most 3 warps, not 7).
#ifndef PREDTOP_ATTN_MINB16
#define PREDTOP_ATTN_MINB16 8  // CTAs per SM of the 4-warp d_h = 16 kernel (register target)
#endif
template <int DH, bool RESIDENT, int NW = 8>
__global__ void __launch_bounds__(NW * 32, (DH == 16 && NW == 4) ? PREDTOP_ATTN_MINB16
                                           : (DH == 16 ? 4 : PREDTOP_ATTN_MINB32) * (8 / NW))
    k_attn(const __grid_constant__ CUtensorMap tkv, DagDev d, int G, int H, int dmodel,
           const __half* __restrict__ qkv, __half* __restrict__ out, int nmax) {
  using A = Attn<DH>;
  constexpr int kStageChunks = stage_chunks<DH>();
  extern __shared__ __align__(16) unsigned char dsm_attn[];
  __shared__ __align__(8) uint64_t kv_full[kStages];
  const int h = blockIdx.x % H;
  const int widx = (blockIdx.x / H) / (8 / NW);
  const int part = (blockIdx.x / H) % (8 / NW);
  if (widx >= d.qtile_off[G]) return;
  const int2 wk = d.work[widx];
  const int g = wk.x, qt = wk.y;
  if ((unsigned)g >= (unsigned)G || d.status[g] != PREDTOP_OK) return;
  const int64_t n0 = d.node_ptr[g];
  const int N = (int)(d.node_ptr[g + 1] - n0);
  if (N > nmax) return;  // a larger graph: the tcgen05 kernel's (attention_tc.cu)
  const int rbase = qt * 128 + part * NW * 16;  // first query row of this CTA
  if (rbase >= N) return;
  const int W = 2 * ((N + 127) / 128);
  const int nchunks = (N + kChunk - 1) / kChunk;
  const int nbuf = RESIDENT ? nchunks : kStages * kStageChunks;
  // K/V chunks (swizzle period <= 512 B: 256-byte alignment suffices for SW32/SW64
  // relative addressing... the resident kernel keeps 1 KB alignment only when
  // the mask staging does not need the room)
  unsigned char* sK = RESIDENT ? sm100::align256(dsm_attn) : sm100::align1024(dsm_attn);
  unsigned char* sV = sK + (size_t)nbuf * A::CHUNK_BYTES;
  // resident path: this CTA's mask rows (NW*16 rows x W words) staged in shared
  // memory by one bulk copy with the K/V, so the per-chunk mask reads in the
  // inner loop are shared-memory loads, not L2 round trips
  unsigned char* sM = sV + (size_t)nbuf * A::CHUNK_BYTES;
  const uint64_t* Mg = d.M + d.row_off[g];
  const int ld3 = 3 * dmodel;
  const __half* Qg = qkv + n0 * ld3 + h * DH;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int gq = lane >> 2, tq = lane & 3;
  const int ra = rbase + warp * 16 + gq;  // graph-local query rows of this thread
  const int rb = ra + 8;
  const bool va = ra < N, vb = rb < N;
  const bool warp_live = rbase + warp * 16 < N;
  const uint64_t* Ma = Mg + (int64_t)(va ? ra : 0) * W;
  const uint64_t* Mb = Mg + (int64_t)(vb ? rb : 0) * W;
  // block flags of this warp's 16-row group, one byte per chunk (k_bflags)
  const uint8_t* Fw = d.bflag + d.bflag_off[g] + (int64_t)(warp_live ? rbase / 16 + warp : 0) * nchunks;

  // K/V chunks by TMA (one thread): [64 keys x DH] boxes of the qkv matrix at
  // columns d + h*DH (K) and 2d + h*DH (V); keys past N read the next graph's
  // rows (masked) or zeros past the tensor end.
  if (threadIdx.x == 0) {
    for (int i = 0; i < kStages; ++i) sm100::mbar_init(&kv_full[i], 1);
    sm100::fence_mbar_init();
  }
  __syncthreads();
  auto load_chunks = [&](int c0, int c1, int slot0, uint64_t* bar) {
    sm100::mbar_arrive_expect_tx(bar, (uint32_t)((c1 - c0) * 2 * A::CHUNK_BYTES));
    for (int c = c0; c < c1; ++c) {
      const int row = (int)(n0 + c * kChunk);
      const int slot = slot0 + c - c0;
      sm100::tma_load_2d(sK + slot * A::CHUNK_BYTES, &tkv, bar, dmodel + h * DH, row);
      sm100::tma_load_2d(sV + slot * A::CHUNK_BYTES, &tkv, bar, 2 * dmodel + h * DH, row);
    }
  };
  if (threadIdx.x == 0) {
    if (RESIDENT) {
      const int rows = min(NW * 16, N - rbase);
      const uint32_t mbytes = (uint32_t)(rows * W * 8);
      sm100::mbar_expect_tx(&kv_full[0], mbytes);
      sm100::bulk_load_1d(sM, Mg + (int64_t)rbase * W, mbytes, &kv_full[0]);
      load_chunks(0, nchunks, 0, &kv_full[0]);
    } else {
      for (int s = 0; s < kStages && s * kStageChunks < nchunks; ++s)
        load_chunks(s * kStageChunks, min(nchunks, (s + 1) * kStageChunks), s * kStageChunks, &kv_full[s]);
    }
  }

  A st;
  st.init(lane);
  uint32_t kw[A::KS][4];
#pragma unroll
  for (int ks = 0; ks < A::KS; ++ks) {
    const int k0 = ks * 16 + 2 * tq;
    const __half* qa_p = Qg + (int64_t)ra * ld3 + k0;
    const __half* qb_p = Qg + (int64_t)rb * ld3 + k0;
    st.qa[ks][0] = va ? *reinterpret_cast<const uint32_t*>(qa_p) : 0u;
    st.qa[ks][1] = vb ? *reinterpret_cast<const uint32_t*>(qb_p) : 0u;
    st.qa[ks][2] = va ? *reinterpret_cast<const uint32_t*>(qa_p + 8) : 0u;
    st.qa[ks][3] = vb ? *reinterpret_cast<const uint32_t*>(qb_p + 8) : 0u;
    kw[ks][0] = va ? *reinterpret_cast<const uint32_t*>(qa_p + dmodel) : 0u;
    kw[ks][1] = vb ? *reinterpret_cast<const uint32_t*>(qb_p + dmodel) : 0u;
    kw[ks][2] = va ? *reinterpret_cast<const uint32_t*>(qa_p + dmodel + 8) : 0u;
    kw[ks][3] = vb ? *reinterpret_cast<const uint32_t*>(qb_p + dmodel + 8) : 0u;
  }
  // reference m of each row: its diagonal score q.k (M includes I, so the
  // row max is >= it; with lazy rescaling m stays within 8 of the max)
  {
    float sa = 0.f, sb = 0.f;
#pragma unroll
    for (int ks = 0; ks < A::KS; ++ks) {
      sa += dot_h2(st.qa[ks][0], kw[ks][0]) + dot_h2(st.qa[ks][2], kw[ks][2]);
      sb += dot_h2(st.qa[ks][1], kw[ks][1]) + dot_h2(st.qa[ks][3], kw[ks][3]);
    }
    sa += __shfl_xor_sync(0xffffffffu, sa, 1);
    sa += __shfl_xor_sync(0xffffffffu, sa, 2);
    sb += __shfl_xor_sync(0xffffffffu, sb, 1);
    sb += __shfl_xor_sync(0xffffffffu, sb, 2);
    st.m_a = sa;
    st.m_b = sb;
  }
  // this thread's 16 mask bits of rows a / b in chunk c: 16-bit piece tq of
  // the (stored-layout) word; raw pieces, combined only where used, so the
  // loads for chunk c+1 are issued before chunk c and hide behind it
  const uint16_t* Ma16 = RESIDENT ? reinterpret_cast<const uint16_t*>(sM + (size_t)(warp * 16 + gq) * W * 8) + tq
                                  : reinterpret_cast<const uint16_t*>(Ma) + tq;
  const uint16_t* Mb16 = RESIDENT ? Ma16 + 8 * W * 4 : reinterpret_cast<const uint16_t*>(Mb) + tq;
  auto mask_lo = [&](int c) -> uint32_t { return va ? (uint32_t)Ma16[4 * c] : 0u; };
  auto mask_hi = [&](int c) -> uint32_t { return vb ? (uint32_t)Mb16[4 * c] : 0u; };
  uint32_t mlo = RESIDENT ? 0u : mask_lo(0), mhi = RESIDENT ? 0u : mask_hi(0);
  const uint32_t kb0 = sm100::smem_u32(sK), vb0 = sm100::smem_u32(sV);

  if (RESIDENT) {
    sm100::mbar_wait(&kv_full[0], 0);
    if (!warp_live) return;
    mlo = mask_lo(0);
    mhi = mask_hi(0);
    uint32_t fl = Fw[0];
    for (int c = 0; c < nchunks; ++c) {
      const bool more = c + 1 < nchunks;
      const uint32_t nlo = more ? mask_lo(c + 1) : 0u, nhi = more ? mask_hi(c + 1) : 0u;
      const uint32_t nfl = more ? Fw[c + 1] : 0u;
      const uint32_t off = (uint32_t)(c * A::CHUNK_BYTES);
      st.chunk(kb0 + off, vb0 + off, mlo | (mhi << 16), __shfl_sync(0xffffffffu, fl, 0));
      mlo = nlo;
      mhi = nhi;
      fl = nfl;
    }
  } else {
    // streaming: a ring of kStages stages of kStageChunks chunks each; stage
    // s+kStages is loaded into the buffer of stage s once every warp is done
    // with it (one CTA barrier per stage), so kStages-1 stages (>= 512 keys)
    // are in flight ahead of the compute and the TMA latency stays hidden
    const int nst = (nchunks + kStageChunks - 1) / kStageChunks;
    for (int s = 0; s < nst; ++s) {
      const int buf = s % kStages;
      const int c0 = s * kStageChunks, c1 = min(nchunks, c0 + kStageChunks);
      sm100::mbar_wait(&kv_full[buf], (s / kStages) & 1);
      for (int c = c0; c < c1; ++c) {
        const bool more = c + 1 < nchunks;
        const uint32_t nlo = more ? mask_lo(c + 1) : 0u, nhi = more ? mask_hi(c + 1) : 0u;
        if (warp_live) {
          const uint32_t off = (uint32_t)((buf * kStageChunks + c - c0) * A::CHUNK_BYTES);
          const uint32_t fl = __shfl_sync(0xffffffffu, (uint32_t)Fw[c], 0);
          st.chunk(kb0 + off, vb0 + off, mlo | (mhi << 16), fl);
        }
        mlo = nlo;
        mhi = nhi;
      }
      __syncthreads();  // every warp is done with buffer buf before it is reloaded
      if (threadIdx.x == 0 && s + kStages < nst) {
        const int n0c = (s + kStages) * kStageChunks;
        load_chunks(n0c, min(nchunks, n0c + kStageChunks), buf * kStageChunks, &kv_full[buf]);
      }
    }
    if (!warp_live) return;
  }
  const float l_a = st.osum[0], l_b = st.osum[2];
  const float ia = l_a > 0.f ? 1.f / l_a : 0.f, ib = l_b > 0.f ? 1.f / l_b : 0.f;
  __half* Og = out + n0 * dmodel + h * DH;
#pragma unroll
  for (int dn = 0; dn < A::DN; ++dn) {
    const int col = dn * 8 + 2 * tq;
    if (va)
      *reinterpret_cast<uint32_t*>(Og + (int64_t)ra * dmodel + col) =
          pack_h2(st.o[dn][0] * ia, st.o[dn][1] * ia);
    if (vb)
      *reinterpret_cast<uint32_t*>(Og + (int64_t)rb * dmodel + col) =
          pack_h2(st.o[dn][2] * ib, st.o[dn][3] * ib);
  }
}

// d_h = 16: graphs above this many nodes take the tcgen05 kernel
constexpr int kTc16Min = 384;

template <int DH>
predtop_status launch_dh(const predtop_dag_s* dag, int d, int H, const __half* qkv, __half* out,
                         cudaStream_t st, unsigned blocks, int nmax) {
  constexpr int CH_BYTES = kChunk * DH * 2;  // one K or V chunk
  const int G = dag->desc.num_graphs;
  // the shared-memory path is sized by the largest graph THIS launch handles
  const int nbig = std::min(std::min(dag->desc.max_nodes, PREDTOP_MAX_NODES), nmax);
  const int maxch = (int)ceil_div(nbig, kChunk);
  const int resident_bytes = 2 * maxch * CH_BYTES + 1024;
  // the 4-warp resident kernel also stages its 64 mask rows (W words each)
  const int wmax = 2 * (int)ceil_div(nbig, 128);
  const int resident4_bytes = 2 * maxch * CH_BYTES + 64 * wmax * 8 + 256;
  CUtensorMap tkv;
  if (!encode_tma_2d(&tkv, qkv, 2, (uint64_t)3 * d, (uint64_t)dag->desc.total_nodes, DH, kChunk))
    return PREDTOP_ERR_CUDA;
  const char* ap = getenv("PREDTOP_ATTN_MODE");  // "8": 8-warp CTAs, default 4-warp
  const bool half_tiles = !(ap && ap[0] == '8');
  if (half_tiles && resident4_bytes <= 28 * 1024) {
    // 4-warp CTAs (half q-tiles), up to 8 per SM (28 KB + 1 KB static each)
    PT_SMEM_ATTR((k_attn<DH, true, 4>), 28 * 1024);
    k_attn<DH, true, 4><<<2 * blocks, 128, resident4_bytes, st>>>(tkv, dag->d, G, H, d, qkv, out, nmax);
  } else if (resident_bytes + 128 * wmax * 8 <= 100 * 1024) {
    PT_SMEM_ATTR((k_attn<DH, true>), 100 * 1024);
    k_attn<DH, true><<<blocks, 256, resident_bytes + 128 * wmax * 8, st>>>(tkv, dag->d, G, H, d, qkv, out, nmax);
  } else {
    constexpr int stream_bytes = 2 * kStages * stage_chunks<DH>() * CH_BYTES + 1024;
    PT_SMEM_ATTR((k_attn<DH, false>), stream_bytes);
    k_attn<DH, false><<<blocks, 256, stream_bytes, st>>>(tkv, dag->d, G, H, d, qkv, out, nmax);
  }
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

}  // namespace

predtop_status attention_launch(const predtop_dag_s* dag, int d, int H, const __half* qkv,
                                __half* out, cudaStream_t st) {
  const int dh = d / H;
  const int64_t blocks = std::max<int64_t>(1, dag->qtiles_bound) * H;
  if (blocks > 0x7fffffff) {
    set_error("too many attention work items");
    return PREDTOP_ERR_TOO_LARGE;
  }
  ProfScope _p(PK_ATTN, st);
  // tcgen05/TMEM kernel (attention_tc.cu) at d_h = 32, where this kernel's
  // mma.sync QK^T + PV demand equals the MUFU rate.  At d_h = 16 the split is
  // per graph: graphs of more than kTc16Min nodes go to the tcgen05 kernel
  // (its per-CTA prologue is amortised over >= 12 key chunks), smaller ones
  // to this kernel, each launch skipping the other's graphs; a batch without
  // large graphs (the GPT config) launches this kernel only.
  // PREDTOP_ATTN_TC=1 / =0 forces one kernel for every graph (parity tests,
  // A/B runs); PREDTOP_ATTN_TC16_MIN overrides the split size.
  const char* tc = getenv("PREDTOP_ATTN_TC");
  const char* t16 = getenv("PREDTOP_ATTN_TC16_MIN");
  const int tc16_min = t16 ? atoi(t16) : kTc16Min;
  int nsplit = dh == 32 ? 0 : (dag->desc.max_nodes > tc16_min ? tc16_min : INT_MAX);  // k_attn takes N <= nsplit
  if (tc && tc[0] == '1') nsplit = 0;
  if (tc && tc[0] == '0') nsplit = INT_MAX;
  if (dh != 16 && dh != 32) {
    set_error("unsupported head dim %d", dh);
    return PREDTOP_ERR_UNSUPPORTED;
  }
  if (nsplit < INT_MAX && attention_tc_supported(dag, d, H)) {
    predtop_status s = attention_tc_launch(dag, d, H, qkv, out, st, nsplit + 1);
    if (s != PREDTOP_OK || nsplit == 0) return s;
  } else {
    nsplit = INT_MAX;
  }
  if (dh == 16) return launch_dh<16>(dag, d, H, qkv, out, st, (unsigned)blocks, nsplit);
  return launch_dh<32>(dag, d, H, qkv, out, st, (unsigned)blocks, nsplit);
}

}  // namespace predtop
