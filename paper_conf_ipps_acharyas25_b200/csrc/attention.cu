// attention.cu -- K6: reachability-masked multi-head attention, Eqn 1
// with V (reading R1):
//     O_h = softmax(Q_h K_h^T / sqrt(d_h) + M) V_h,  M(u,v) = 0 iff the mask
//     bit M[u][v] of  M = R | R^T | I  is set (DAGRA), else -inf.
//
// One CTA = one (graph, 128-row query tile, head); 8 warps x 16 query rows.
// The 1-D grid runs the heads of a q-tile back to back, so the q/k/v rows of
// a graph are fetched from HBM once and re-read by the other heads from L2.
// Keys/values stream through shared memory in 64-key chunks (cp.async double
// buffer); a chunk is exactly one 64-bit word of each mask row.  Block
// sparsity is exploited per warp at 16-key granularity: a 16 x 16 block whose
// mask bits are all zero for the warp's 16 rows costs no MMA and no exp.
// Online softmax in fp32 with exp2 (MUFU ex2), P rounded once to fp16.
//
// At d_h = 16/32 the kernel is bound by the exponentials (one MUFU ex2 per
// computed score), not by the tensor pipe: QK^T and PV are 2*d_h flops per
// score each.  The warp-level m16n8k16 MMA keeps S and P in registers (the S
// accumulator fragment is the P operand fragment); see DESIGN.md "K6".
#include "internal.h"

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

__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src, bool valid) {
  const int n = valid ? 16 : 0;  // src-size 0 -> zero fill
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(n));
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;"); }
template <int N>
__device__ __forceinline__ void cp_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N));
}

__device__ __forceinline__ uint32_t pack_h2(float a, float b) {
  __half2 h = __floats2half2_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}

constexpr int kChunk = 64;

template <int DH>
__global__ void __launch_bounds__(256, 2) k_attn(DagDev d, int G, int H, int dmodel,
                                                 const __half* __restrict__ qkv,
                                                 __half* __restrict__ out) {
  constexpr int PITCH = DH + 8;  // halves; 48 B / 80 B rows: conflict-free ldmatrix
  constexpr int KS = DH / 16;    // k-steps for QK^T
  constexpr int DN = DH / 8;     // n-tiles of the output
  __shared__ __align__(16) __half sK[2][kChunk * PITCH];
  __shared__ __align__(16) __half sV[2][kChunk * PITCH];

  const int h = blockIdx.x % H;
  const int widx = blockIdx.x / H;
  if (widx >= d.qtile_off[G]) return;
  const int2 wk = d.work[widx];
  const int g = wk.x, qt = wk.y;
  if (d.status[g] != PREDTOP_OK) return;
  const int64_t n0 = d.node_ptr[g];
  const int N = (int)(d.node_ptr[g + 1] - n0);
  const int W = 2 * ((N + 127) / 128);
  const uint64_t* Mg = d.M + d.row_off[g];
  const int ld3 = 3 * dmodel;
  const __half* Qg = qkv + n0 * ld3 + h * DH;
  const __half* Kg = Qg + dmodel;
  const __half* Vg = Qg + 2 * dmodel;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int gq = lane >> 2, tq = lane & 3;
  const int ra = qt * 128 + warp * 16 + gq;  // graph-local query rows of this thread
  const int rb = ra + 8;
  const bool va = ra < N, vb = rb < N;
  const uint64_t* Ma = Mg + (int64_t)(va ? ra : 0) * W;
  const uint64_t* Mb = Mg + (int64_t)(vb ? rb : 0) * W;

  const int nchunks = (N + kChunk - 1) / kChunk;
  constexpr int SEGS = kChunk * DH / 8;  // 16-byte segments per matrix per chunk
  auto load_chunk = [&](int c, int buf) {
    for (int s = threadIdx.x; s < 2 * SEGS; s += blockDim.x) {
      const int mat = s / SEGS, r = (s % SEGS) / (DH / 8), seg = s % (DH / 8);
      const int key = c * kChunk + r;
      const __half* src = (mat ? Vg : Kg) + (int64_t)(key < N ? key : 0) * ld3 + seg * 8;
      __half* dst = (mat ? sV[buf] : sK[buf]) + r * PITCH + seg * 8;
      cp_async16(static_cast<uint32_t>(__cvta_generic_to_shared(dst)), src, key < N);
    }
    cp_commit();
  };
  load_chunk(0, 0);

  // Q fragments (A operand, row-major 16 x 16 per k-step)
  uint32_t qa[KS][4];
#pragma unroll
  for (int ks = 0; ks < KS; ++ks) {
    const int k0 = ks * 16 + 2 * tq;
    qa[ks][0] = va ? *reinterpret_cast<const uint32_t*>(Qg + (int64_t)ra * ld3 + k0) : 0u;
    qa[ks][1] = vb ? *reinterpret_cast<const uint32_t*>(Qg + (int64_t)rb * ld3 + k0) : 0u;
    qa[ks][2] = va ? *reinterpret_cast<const uint32_t*>(Qg + (int64_t)ra * ld3 + k0 + 8) : 0u;
    qa[ks][3] = vb ? *reinterpret_cast<const uint32_t*>(Qg + (int64_t)rb * ld3 + k0 + 8) : 0u;
  }
  const float scale = 1.4426950408889634f * rsqrtf((float)DH);  // log2(e)/sqrt(d_h)

  float o[DN][4];
#pragma unroll
  for (int i = 0; i < DN; ++i) o[i][0] = o[i][1] = o[i][2] = o[i][3] = 0.f;
  float m_a = -INFINITY, m_b = -INFINITY, l_a = 0.f, l_b = 0.f;  // running max (scaled)
  uint64_t mwa = va ? Ma[0] : 0ull, mwb = vb ? Mb[0] : 0ull;

  for (int c = 0; c < nchunks; ++c) {
    const int buf = c & 1;
    // prefetch the next chunk's K/V and mask words
    uint64_t nwa = 0ull, nwb = 0ull;
    if (c + 1 < nchunks) {
      load_chunk(c + 1, buf ^ 1);
      nwa = va ? Ma[c + 1] : 0ull;
      nwb = vb ? Mb[c + 1] : 0ull;
      cp_wait<1>();
    } else {
      cp_wait<0>();
    }
    __syncthreads();
    // 16-key blocks with at least one allowed pair among the warp's 16 rows
    uint32_t act = 0;
#pragma unroll
    for (int j = 0; j < 4; ++j)
      act |= __any_sync(0xffffffffu, ((mwa | mwb) >> (16 * j)) & 0xffffull) ? (1u << j) : 0u;
    if (act) {
      const uint32_t kbase = static_cast<uint32_t>(__cvta_generic_to_shared(sK[buf]));
      const uint32_t vbase = static_cast<uint32_t>(__cvta_generic_to_shared(sV[buf]));
      float s[8][4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          s[2 * j + u][0] = s[2 * j + u][1] = s[2 * j + u][2] = s[2 * j + u][3] = 0.f;
        }
        if (act & (1u << j)) {
#pragma unroll
          for (int ks = 0; ks < KS; ++ks) {
            // x4: matrices = (keys 16j+0..7, dims lo), (keys 16j+0..7, dims hi),
            //                (keys 16j+8..15, dims lo), (keys 16j+8..15, dims hi)
            const int r = 16 * j + ((lane >> 4) & 1) * 8 + (lane & 7);
            const int col = ks * 16 + ((lane >> 3) & 1) * 8;
            uint32_t b0, b1, b2, b3;
            ldsm_x4(kbase + (uint32_t)((r * PITCH + col) * 2), b0, b1, b2, b3);
            mma16816(s[2 * j], qa[ks], b0, b1);
            mma16816(s[2 * j + 1], qa[ks], b2, b3);
          }
        }
      }
      // masked running max over raw scores
      float mx_a = -INFINITY, mx_b = -INFINITY;
#pragma unroll
      for (int nt = 0; nt < 8; ++nt) {
        const int bit = nt * 8 + 2 * tq;
        if (act & (1u << (nt >> 1))) {
          if ((mwa >> bit) & 1ull) mx_a = fmaxf(mx_a, s[nt][0]);
          if ((mwa >> (bit + 1)) & 1ull) mx_a = fmaxf(mx_a, s[nt][1]);
          if ((mwb >> bit) & 1ull) mx_b = fmaxf(mx_b, s[nt][2]);
          if ((mwb >> (bit + 1)) & 1ull) mx_b = fmaxf(mx_b, s[nt][3]);
        }
      }
      mx_a = fmaxf(mx_a, __shfl_xor_sync(0xffffffffu, mx_a, 1));
      mx_a = fmaxf(mx_a, __shfl_xor_sync(0xffffffffu, mx_a, 2));
      mx_b = fmaxf(mx_b, __shfl_xor_sync(0xffffffffu, mx_b, 1));
      mx_b = fmaxf(mx_b, __shfl_xor_sync(0xffffffffu, mx_b, 2));
      const float mn_a = fmaxf(m_a, mx_a * scale), mn_b = fmaxf(m_b, mx_b * scale);
      const float mu_a = mn_a == -INFINITY ? 0.f : mn_a;
      const float mu_b = mn_b == -INFINITY ? 0.f : mn_b;
      const float al_a = ex2(m_a - mu_a), al_b = ex2(m_b - mu_b);
      m_a = mn_a;
      m_b = mn_b;
      l_a *= al_a;
      l_b *= al_b;
#pragma unroll
      for (int i = 0; i < DN; ++i) {
        o[i][0] *= al_a; o[i][1] *= al_a;
        o[i][2] *= al_b; o[i][3] *= al_b;
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        if (!(act & (1u << j))) continue;
        uint32_t pa[4];
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          const int nt = 2 * j + u;
          const int bit = nt * 8 + 2 * tq;
          float p0 = ex2(fmaf(s[nt][0], scale, -mu_a));
          float p1 = ex2(fmaf(s[nt][1], scale, -mu_a));
          float p2 = ex2(fmaf(s[nt][2], scale, -mu_b));
          float p3 = ex2(fmaf(s[nt][3], scale, -mu_b));
          p0 = ((mwa >> bit) & 1ull) ? p0 : 0.f;
          p1 = ((mwa >> (bit + 1)) & 1ull) ? p1 : 0.f;
          p2 = ((mwb >> bit) & 1ull) ? p2 : 0.f;
          p3 = ((mwb >> (bit + 1)) & 1ull) ? p3 : 0.f;
          l_a += p0 + p1;
          l_b += p2 + p3;
          pa[2 * u + 0] = pack_h2(p0, p1);
          pa[2 * u + 1] = pack_h2(p2, p3);
        }
        // PV: B = V[keys 16j..16j+15][dims], transposed ldmatrix; x4 covers two
        // 8-dim n-tiles: (keys lo, dims 8m..), (keys hi, dims 8m..), (keys lo, dims 8m+8..), ...
#pragma unroll
        for (int dn = 0; dn < DN; dn += 2) {
          const int r = 16 * j + ((lane >> 3) & 1) * 8 + (lane & 7);
          const int col = dn * 8 + ((lane >> 4) & 1) * 8;
          uint32_t b0, b1, b2, b3;
          ldsm_x4_t(vbase + (uint32_t)((r * PITCH + col) * 2), b0, b1, b2, b3);
          mma16816(o[dn], pa, b0, b1);
          mma16816(o[dn + 1], pa, b2, b3);
        }
      }
    }
    __syncthreads();
    mwa = nwa;
    mwb = nwb;
  }
  l_a += __shfl_xor_sync(0xffffffffu, l_a, 1);
  l_a += __shfl_xor_sync(0xffffffffu, l_a, 2);
  l_b += __shfl_xor_sync(0xffffffffu, l_b, 1);
  l_b += __shfl_xor_sync(0xffffffffu, l_b, 2);
  const float ia = l_a > 0.f ? 1.f / l_a : 0.f, ib = l_b > 0.f ? 1.f / l_b : 0.f;
  __half* Og = out + n0 * dmodel + h * DH;
#pragma unroll
  for (int dn = 0; dn < DN; ++dn) {
    const int col = dn * 8 + 2 * tq;
    if (va)
      *reinterpret_cast<uint32_t*>(Og + (int64_t)ra * dmodel + col) = pack_h2(o[dn][0] * ia, o[dn][1] * ia);
    if (vb)
      *reinterpret_cast<uint32_t*>(Og + (int64_t)rb * dmodel + col) = pack_h2(o[dn][2] * ib, o[dn][3] * ib);
  }
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
  const int G = dag->desc.num_graphs;
  ProfScope _p(PK_ATTN, st);
  if (dh == 16) k_attn<16><<<(unsigned)blocks, 256, 0, st>>>(dag->d, G, H, d, qkv, out);
  else if (dh == 32) k_attn<32><<<(unsigned)blocks, 256, 0, st>>>(dag->d, G, H, d, qkv, out);
  else {
    set_error("unsupported head dim %d", dh);
    return PREDTOP_ERR_UNSUPPORTED;
  }
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

}  // namespace predtop
