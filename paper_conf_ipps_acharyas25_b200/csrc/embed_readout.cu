// embed_readout.cu -- node embedding (Table I features + DAGPE) and the
// graph readout (global add pool + MLP head), both fp32 on CUDA cores.
//
// K4  x0[v] = b_in + W_in[:,op] + sum_j ln(1+dims_j) W_in[:,64+j]
//           + W_in[:,68+dtype] + W_in[:,76+kind] + PE(depth v)
//     (Table I; log scaling P:167; DAGPE P:137, sinusoidal PE of
//      [34] over the depth, reading R5).  The one-hot product is a row gather
//      of the transposed W_in; the PE comes from a per-call table indexed by
//      depth, computed in fp64 (angles up to ~1e4 rad for deep graphs).
// K8  g = sum_n x_n (Eqn 2; mean if pool = MEAN), then
//     y = w_o . ReLU(H_2 ReLU(H_1 g + c_1) + c_2) + c_o
//     One CTA per graph, fixed summation order: deterministic per graph.
#include "internal.h"

namespace predtop {

__global__ void k_pe_table(float* pe, int rows, int d) {
  const int half = d / 2;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (int64_t)rows * half;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int depth = (int)(i / half), k = (int)(i % half);
    const double w = pow(10000.0, -(2.0 * k) / d);
    double s, c;
    sincos((double)depth * w, &s, &c);
    pe[(int64_t)depth * d + 2 * k] = (float)s;
    pe[(int64_t)depth * d + 2 * k + 1] = (float)c;
  }
}

predtop_status pe_table_launch(float* pe, int rows, int d, cudaStream_t st) {
  const int64_t n = (int64_t)rows * (d / 2);
  const int blocks = (int)std::min<int64_t>(ceil_div(n, 256), 148 * 8);
{
    ProfScope _p(PK_PE, st);
    k_pe_table<<<blocks, 256, 0, st>>>(pe, rows, d);
    PT_LAUNCH_CHECK();
  }
  return PREDTOP_OK;
}

// A lane's PER columns of a D-wide fp32 row: groups of four at columns
// 4 lane + 128 j (each 16-byte vector instruction of the warp covers 512
// contiguous bytes), or PER < 4 consecutive columns at PER lane.
template <int PER>
__device__ __forceinline__ int col_of(int lane, int k) {
  if constexpr (PER >= 4) return 128 * (k / 4) + 4 * lane + (k % 4);
  else return PER * lane + k;
}
template <int PER>
__device__ __forceinline__ void ld_cols(const float* __restrict__ row, int lane, float (&a)[PER]) {
  if constexpr (PER % 4 == 0) {
#pragma unroll
    for (int j = 0; j < PER / 4; ++j) {
      const float4 v = __ldg(reinterpret_cast<const float4*>(row + 128 * j + 4 * lane));
      a[4 * j] = v.x, a[4 * j + 1] = v.y, a[4 * j + 2] = v.z, a[4 * j + 3] = v.w;
    }
  } else if constexpr (PER == 2) {
    const float2 v = __ldg(reinterpret_cast<const float2*>(row + 2 * lane));
    a[0] = v.x, a[1] = v.y;
  } else {
#pragma unroll
    for (int k = 0; k < PER; ++k) a[k] = __ldg(row + PER * lane + k);
  }
}

template <int D>
__global__ void __launch_bounds__(256, 4) k_embed(const float* __restrict__ WT, const float* __restrict__ b,
                                               const predtop_node_feat* __restrict__ feats,
                                               const int32_t* __restrict__ depth,
                                               const float* __restrict__ pe, int pe_rows, int64_t n_tot,
                                               float* __restrict__ x32, __half* __restrict__ x16) {
  // one warp per node, PER = D / 32 columns per lane (col_of: vector loads of
  // the W_in^T rows and the PE row, coalesced vector stores)
  constexpr int PER = D / 32;
  const int lane = threadIdx.x & 31;
  const int64_t warp0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  float bias[PER];
  ld_cols<PER>(b, lane, bias);
  // the next node's features and depth are loaded one iteration ahead (the
  // row gathers depend on them: two dependent round trips per node otherwise)
  predtop_node_feat fn{};
  int dn = 0;
  if (warp0 < n_tot) {
    fn = feats[warp0];
    dn = depth[warp0];
  }
  for (int64_t v = warp0; v < n_tot; v += nwarps) {
    const predtop_node_feat f = fn;
    // a graph with an error status (latency NaN) may hold no depth at all
    // (TOO_LARGE / INVALID_ARG graphs are never built): clamp into the table
    const int dep = min(max(dn, 0), pe_rows - 1);
    if (v + nwarps < n_tot) {
      fn = feats[v + nwarps];
      dn = depth[v + nwarps];
    }
    float acc[PER], t[PER];
#pragma unroll
    for (int k = 0; k < PER; ++k) acc[k] = bias[k];
    if (f.op < PREDTOP_NUM_OPS) {
      ld_cols<PER>(WT + (size_t)f.op * D, lane, t);
#pragma unroll
      for (int k = 0; k < PER; ++k) acc[k] += t[k];
    }
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const float l = log1pf((float)f.dims[j]);
      ld_cols<PER>(WT + (size_t)(64 + j) * D, lane, t);
#pragma unroll
      for (int k = 0; k < PER; ++k) acc[k] += l * t[k];
    }
    if (f.dtype < PREDTOP_NUM_DTYPES) {
      ld_cols<PER>(WT + (size_t)(68 + f.dtype) * D, lane, t);
#pragma unroll
      for (int k = 0; k < PER; ++k) acc[k] += t[k];
    }
    if (f.kind < PREDTOP_NUM_KINDS) {
      ld_cols<PER>(WT + (size_t)(76 + f.kind) * D, lane, t);
#pragma unroll
      for (int k = 0; k < PER; ++k) acc[k] += t[k];
    }
    ld_cols<PER>(pe + (size_t)dep * D, lane, t);
#pragma unroll
    for (int k = 0; k < PER; ++k) acc[k] += t[k];
    float* o32 = x32 + v * D;
    __half* o16 = x16 + v * D;
    if constexpr (PER % 4 == 0) {
#pragma unroll
      for (int j = 0; j < PER / 4; ++j) {
        const int c = 128 * j + 4 * lane;
        *reinterpret_cast<float4*>(o32 + c) = make_float4(acc[4 * j], acc[4 * j + 1], acc[4 * j + 2], acc[4 * j + 3]);
        __half2 h[2] = {__floats2half2_rn(acc[4 * j], acc[4 * j + 1]), __floats2half2_rn(acc[4 * j + 2], acc[4 * j + 3])};
        *reinterpret_cast<uint2*>(o16 + c) = *reinterpret_cast<const uint2*>(h);
      }
    } else {
#pragma unroll
      for (int k = 0; k < PER; ++k) {
        o32[col_of<PER>(lane, k)] = acc[k];
        o16[col_of<PER>(lane, k)] = __float2half_rn(acc[k]);
      }
    }
  }
}

predtop_status embed_launch(const predtop_model_s* m, const predtop_dag_s* dag, const float* pe,
                            float* x32, __half* x16, cudaStream_t st) {
  const int64_t n = dag->desc.total_nodes;
  const int blocks = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 8), 148 * 16));
  const DagDev& d = dag->d;
  const int pe_rows = std::min<int>(dag->desc.max_nodes, PREDTOP_MAX_NODES);
  ProfScope _p(PK_EMBED, st);
#define PT_EMBED(D)                                                                  \
  case D:                                                                            \
    k_embed<D><<<blocks, 256, 0, st>>>(m->W_inT, m->b_in, d.feats, d.depth, pe, pe_rows, n, x32, x16); \
    break;
  switch (m->cfg.d_model) {
    PT_EMBED(32)
    PT_EMBED(64)
    PT_EMBED(128)
    PT_EMBED(256)
    default: set_error("unsupported d_model"); return PREDTOP_ERR_UNSUPPORTED;
  }
#undef PT_EMBED
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

// ---------------------------------------------------------------- readout
template <int D>
__global__ void __launch_bounds__(D) k_readout(const float* __restrict__ x32,
                                               const int64_t* __restrict__ node_ptr,
                                               const int32_t* __restrict__ status, int pool_mean,
                                               const float* __restrict__ H1T, const float* __restrict__ c1,
                                               const float* __restrict__ H2T, const float* __restrict__ c2,
                                               const float* __restrict__ w_o, const float* __restrict__ c_o,
                                               float* __restrict__ latency) {
  __shared__ float sg[D], sz[D], red[D / 32];
  const int g = blockIdx.x, c = threadIdx.x;
  if (status[g] != PREDTOP_OK) {
    if (c == 0) latency[g] = __int_as_float(0x7fc00000);  // NaN
    return;
  }
  const int64_t n0 = node_ptr[g], n1 = node_ptr[g + 1];
  // Eqn 2: eight interleaved partial sums (node v into partial (v - n0) % 8,
  // combined pairwise in a fixed order: deterministic, and eight independent
  // row loads in flight per thread instead of one dependent add chain)
  float ps[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
  int64_t v = n0;
  for (; v + 8 <= n1; v += 8) {
#pragma unroll
    for (int k = 0; k < 8; ++k) ps[k] += __ldg(x32 + (v + k) * D + c);
  }
  for (int k = 0; v < n1; ++v, ++k) ps[k] += __ldg(x32 + v * D + c);
  float s = ((ps[0] + ps[1]) + (ps[2] + ps[3])) + ((ps[4] + ps[5]) + (ps[6] + ps[7]));
  if (pool_mean) s /= (float)(n1 - n0);
  sg[c] = s;
  __syncthreads();
  float z = c1[c];
  for (int i = 0; i < D; ++i) z += H1T[i * D + c] * sg[i];
  sz[c] = fmaxf(z, 0.f);
  __syncthreads();
  z = c2[c];
  for (int i = 0; i < D; ++i) z += H2T[i * D + c] * sz[i];
  z = fmaxf(z, 0.f);
  float p = w_o[c] * z;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) p += __shfl_xor_sync(0xffffffffu, p, o);
  if ((c & 31) == 0) red[c >> 5] = p;
  __syncthreads();
  if (c == 0) {
    float y = 0.f;
    for (int w = 0; w < D / 32; ++w) y += red[w];
    latency[g] = y + c_o[0];
  }
}

predtop_status readout_launch(const predtop_model_s* m, const predtop_dag_s* dag, const float* x32,
                              float* latency, cudaStream_t st) {
  const int G = dag->desc.num_graphs;
  const DagDev& d = dag->d;
  ProfScope _p(PK_READOUT, st);
#define PT_READ(D)                                                                       \
  case D:                                                                                \
    k_readout<D><<<G, D, 0, st>>>(x32, d.node_ptr, d.status, m->cfg.pool, m->H1T, m->c1, \
                                  m->H2T, m->c2, m->w_o, m->c_o, latency);               \
    break;
  switch (m->cfg.d_model) {
    PT_READ(32)
    PT_READ(64)
    PT_READ(128)
    PT_READ(256)
    default: set_error("unsupported d_model"); return PREDTOP_ERR_UNSUPPORTED;
  }
#undef PT_READ
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

}  // namespace predtop
