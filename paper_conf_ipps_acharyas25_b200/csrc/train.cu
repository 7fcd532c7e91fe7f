// train.cu -- SURVEY 8(f) f4: training of the DAG-Transformer latency model
// (SIV-B6-8; the training phase of P:219).
//
// One predtop_train_grad call = fp32 forward over a batch of stage DAGs with
// every activation kept, the MAE loss of Eqn 3, and the reverse of
// every forward step (K4 embedding, K5 QKV, K6 masked attention, K7 O-proj +
// LN + FFN + LN, K8 pool + head) into a gradient blob laid out like the
// weight blob; predtop_train_adam applies Adam.  Readings R1-R11 as
// in the inference path (include/predtop.h), all in fp32: no fp16 operands,
// since gradients of a regression model trained from scratch need the range.
//
// Dense products (all the Linear layers, forward and backward) are plain
// cuBLAS SGEMMs (fp32, no TF32).  The masked attention keeps its probability
// matrices P (per layer, graph, head: N_g^2 floats at offset
// (tile_off[g] H + h T_g^2) * 128^2 -- T_g = ceil(N_g/128), so the build's
// tile prefix sizes them) and runs one warp per (query row, head): scores on
// the allowed keys (mask bit of the stored layout), max, exp, sum, P row, then
// O = P V with lane j on dimension j.  The backward splits rows and keys so
// that nothing needs float atomics:
//   rows  (warp per (u, h)): dP_uv = dO_u . V_v, D_u = sum_v P_uv dP_uv,
//                            dS_uv = P_uv (dP_uv - D_u), dQ_u = dS_u K / sqrt(d_h)
//   keys  (warp per (v, h)): dV_v = sum_u P_uv dO_u, dK_v = sum_u dS_uv Q_u / sqrt(d_h)
// Column sums (bias and LayerNorm parameter gradients) use one thread per
// column over the rows in fixed order: deterministic.
#include <cublas_v2.h>

#include <algorithm>
#include <cmath>

#include "internal.h"

struct predtop_train_s {
  predtop_model_config cfg;
  int64_t nparam;
  float* buf[4];  // params, grad, m, v
  cublasHandle_t blas;
  int device;
};

namespace predtop {
namespace {

constexpr int kF = PREDTOP_NUM_FEATURES;

// offsets (floats) of every tensor in the weight blob
struct Offs {
  int64_t W_in, b_in, H1, c1, H2, c2, w_o, c_o, total;
  struct L {
    int64_t Wqkv, bqkv, Wo, bo, g1, be1, W1, b1, W2, b2, g2, be2;
  } l[kMaxLayers];
};
Offs offsets(const predtop_model_config& c) {
  const int64_t d = c.d_model, f = c.d_ff;
  Offs o{};
  int64_t p = 0;
  o.W_in = p; p += d * kF;
  o.b_in = p; p += d;
  for (int l = 0; l < c.num_layers; ++l) {
    auto& L = o.l[l];
    L.Wqkv = p; p += 3 * d * d;
    L.bqkv = p; p += 3 * d;
    L.Wo = p; p += d * d;
    L.bo = p; p += d;
    L.g1 = p; p += d;
    L.be1 = p; p += d;
    L.W1 = p; p += f * d;
    L.b1 = p; p += f;
    L.W2 = p; p += d * f;
    L.b2 = p; p += d;
    L.g2 = p; p += d;
    L.be2 = p; p += d;
  }
  o.H1 = p; p += d * d;
  o.c1 = p; p += d;
  o.H2 = p; p += d * d;
  o.c2 = p; p += d;
  o.w_o = p; p += d;
  o.c_o = p; p += 1;
  o.total = p;
  return o;
}

bool train_cfg_ok(const predtop_model_config* c) {
  return c && c->num_layers >= 1 && c->num_layers <= kMaxLayers && c->d_model >= 2 && c->d_model <= 256 &&
         c->d_model % 2 == 0 && c->num_heads >= 1 && c->d_model % c->num_heads == 0 &&
         c->d_model / c->num_heads <= 32 && c->d_ff >= 1 && c->d_ff <= 4096 &&
         (c->pool == PREDTOP_POOL_SUM || c->pool == PREDTOP_POOL_MEAN) && c->ln_eps > 0.f;
}

// ---------------------------------------------------------------- cuBLAS
// Row-major C[M x N] = alpha op(A) op(B) + beta C, op(A) M x K, op(B) K x N
// (column-major identity C^T = op(B)^T op(A)^T).
cublasStatus_t gemm(cublasHandle_t h, bool ta, bool tb, int M, int N, int K, const float* A, int lda,
                    const float* B, int ldb, float beta, float* C, int ldc, float alpha = 1.f) {
  return cublasSgemm(h, tb ? CUBLAS_OP_T : CUBLAS_OP_N, ta ? CUBLAS_OP_T : CUBLAS_OP_N, N, M, K, &alpha, B, ldb,
                     A, lda, &beta, C, ldc);
}
#define PT_BLAS(expr)                                                          \
  do {                                                                         \
    cublasStatus_t _b = (expr);                                                \
    note_launch();                                                             \
    if (_b != CUBLAS_STATUS_SUCCESS) {                                         \
      set_error("cuBLAS %s failed (%d) (%s:%d)", #expr, (int)_b, __FILE__, __LINE__); \
      return PREDTOP_ERR_CUDA;                                                 \
    }                                                                          \
  } while (0)

// ---------------------------------------------------------------- kernels
__global__ void k_tr_gid(const int64_t* __restrict__ node_ptr, int G, int32_t* __restrict__ gid) {
  for (int g = blockIdx.x; g < G; g += gridDim.x)
    for (int64_t v = node_ptr[g] + threadIdx.x; v < node_ptr[g + 1]; v += blockDim.x) gid[v] = g;
}

// dense Table I features (reading R9) [N][F]
__global__ void k_tr_features(const predtop_node_feat* __restrict__ feats, int64_t N, float* __restrict__ F) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N * kF; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = i / kF;
    const int f = (int)(i % kF);
    const predtop_node_feat r = feats[v];
    float x = 0.f;
    if (f < PREDTOP_NUM_OPS) x = r.op == f ? 1.f : 0.f;
    else if (f < PREDTOP_NUM_OPS + 4) x = log1pf((float)r.dims[f - PREDTOP_NUM_OPS]);
    else if (f < PREDTOP_NUM_OPS + 4 + PREDTOP_NUM_DTYPES) x = r.dtype == f - PREDTOP_NUM_OPS - 4 ? 1.f : 0.f;
    else x = r.kind == f - PREDTOP_NUM_OPS - 4 - PREDTOP_NUM_DTYPES ? 1.f : 0.f;
    F[i] = x;
  }
}

// C[r][c] = bias[c] (+ R[r][c]): the initial value of a GEMM accumulated with beta = 1
__global__ void k_tr_init_rows(float* __restrict__ C, const float* __restrict__ bias, const float* __restrict__ R,
                               int64_t rows, int cols) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < rows * cols; i += (int64_t)gridDim.x * blockDim.x)
    C[i] = (bias ? bias[i % cols] : 0.f) + (R ? R[i] : 0.f);
}

// x0 += b_in + PE(depth) (reading R5: sin/cos of depth * 10000^(-2i/d))
__global__ void k_tr_embed_finish(float* __restrict__ x, const float* __restrict__ b_in, const int32_t* __restrict__ depth,
                                  int64_t N, int d) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N * d; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = i / d;
    const int c = (int)(i % d);
    const double w = pow(10000.0, -(double)(c & ~1) / d);
    const double a = (double)depth[v] * w;
    x[i] += b_in[c] + (float)((c & 1) ? cos(a) : sin(a));
  }
}

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

struct AttnView {
  const int64_t* node_ptr;
  const int64_t* row_off;
  const int64_t* tile_off;
  const uint64_t* M;  // stored layout (internal.h mask_pos)
  const int32_t* gid;
  int H, d, dh;
  float scale;        // 1 / sqrt(d_h)
};
__device__ __forceinline__ bool allowed(const uint64_t* Mrow, int k) {
  return (Mrow[k >> 6] >> mask_pos(k & 63)) & 1ull;
}
__device__ __forceinline__ float* p_row(float* P, const AttnView& a, int g, int h, int N, int u) {
  const int T = (N + 127) / 128;
  return P + ((a.tile_off[g] * a.H + (int64_t)h * T * T) << 14) + (int64_t)u * N;
}

// Eqn 1 forward, warp per (node, head); saves P
__global__ void k_tr_attn_fwd(AttnView a, int64_t Ntot, const float* __restrict__ qkv, float* __restrict__ P,
                              float* __restrict__ out) {
  const int64_t wid = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (wid >= Ntot * a.H) return;
  const int64_t v = wid / a.H;
  const int h = (int)(wid % a.H);
  const int g = a.gid[v];
  const int64_t n0 = a.node_ptr[g];
  const int N = (int)(a.node_ptr[g + 1] - n0);
  const int u = (int)(v - n0);
  const int W = 2 * ((N + 127) / 128);
  const uint64_t* Mrow = a.M + a.row_off[g] + (int64_t)u * W;
  float q[32];
#pragma unroll
  for (int j = 0; j < 32; ++j) q[j] = j < a.dh ? qkv[v * 3 * a.d + h * a.dh + j] : 0.f;
  float* Pr = p_row(P, a, g, h, N, u);
  float mx = -INFINITY;
  for (int k = lane; k < N; k += 32) {
    float s = -INFINITY;
    if (allowed(Mrow, k)) {
      const float* kr = qkv + (n0 + k) * 3 * a.d + a.d + h * a.dh;
      s = 0.f;
      for (int j = 0; j < a.dh; ++j) s = fmaf(q[j], kr[j], s);
      s *= a.scale;
    }
    Pr[k] = s;
    mx = fmaxf(mx, s);
  }
  mx = warp_max(mx);
  float sum = 0.f;
  for (int k = lane; k < N; k += 32) {
    const float e = Pr[k] == -INFINITY ? 0.f : expf(Pr[k] - mx);
    Pr[k] = e;
    sum += e;
  }
  sum = warp_sum(sum);
  const float inv = 1.f / sum;
  for (int k = lane; k < N; k += 32) Pr[k] *= inv;
  __syncwarp();
  if (lane < a.dh) {
    float o = 0.f;
    for (int k = 0; k < N; ++k) o = fmaf(Pr[k], qkv[(n0 + k) * 3 * a.d + 2 * a.d + h * a.dh + lane], o);
    out[v * a.d + h * a.dh + lane] = o;
  }
}

// backward, rows: dS (saved) and dQ
__global__ void k_tr_attn_bwd_rows(AttnView a, int64_t Ntot, const float* __restrict__ qkv, const float* __restrict__ P,
                                   const float* __restrict__ dO, float* __restrict__ dS, float* __restrict__ dqkv) {
  const int64_t wid = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (wid >= Ntot * a.H) return;
  const int64_t v = wid / a.H;
  const int h = (int)(wid % a.H);
  const int g = a.gid[v];
  const int64_t n0 = a.node_ptr[g];
  const int N = (int)(a.node_ptr[g + 1] - n0);
  const int u = (int)(v - n0);
  float go[32];
#pragma unroll
  for (int j = 0; j < 32; ++j) go[j] = j < a.dh ? dO[v * a.d + h * a.dh + j] : 0.f;
  const float* Pr = p_row(const_cast<float*>(P), a, g, h, N, u);
  float* Sr = p_row(dS, a, g, h, N, u);
  float D = 0.f;
  for (int k = lane; k < N; k += 32) {
    const float p = Pr[k];
    float dp = 0.f;
    if (p != 0.f) {
      const float* vr = qkv + (n0 + k) * 3 * a.d + 2 * a.d + h * a.dh;
      for (int j = 0; j < a.dh; ++j) dp = fmaf(go[j], vr[j], dp);
    }
    Sr[k] = dp;
    D = fmaf(p, dp, D);
  }
  D = warp_sum(D);
  for (int k = lane; k < N; k += 32) Sr[k] = Pr[k] * (Sr[k] - D);
  __syncwarp();
  if (lane < a.dh) {
    float q = 0.f;
    for (int k = 0; k < N; ++k) q = fmaf(Sr[k], qkv[(n0 + k) * 3 * a.d + a.d + h * a.dh + lane], q);
    dqkv[v * 3 * a.d + h * a.dh + lane] = q * a.scale;
  }
}

// backward, keys: dK, dV (column walks of P and dS)
__global__ void k_tr_attn_bwd_keys(AttnView a, int64_t Ntot, const float* __restrict__ qkv, const float* __restrict__ P,
                                   const float* __restrict__ dS, const float* __restrict__ dO, float* __restrict__ dqkv) {
  const int64_t wid = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (wid >= Ntot * a.H) return;
  const int64_t v = wid / a.H;
  const int h = (int)(wid % a.H);
  const int g = a.gid[v];
  const int64_t n0 = a.node_ptr[g];
  const int N = (int)(a.node_ptr[g + 1] - n0);
  const int w = (int)(v - n0);
  const float* P0 = p_row(const_cast<float*>(P), a, g, h, N, 0);
  const float* S0 = p_row(const_cast<float*>(dS), a, g, h, N, 0);
  if (lane < a.dh) {
    float dv = 0.f, dk = 0.f;
    for (int u = 0; u < N; ++u) {
      const float p = P0[(int64_t)u * N + w];
      if (p == 0.f) continue;  // masked pair (P and dS both zero)
      dv = fmaf(p, dO[(n0 + u) * a.d + h * a.dh + lane], dv);
      dk = fmaf(S0[(int64_t)u * N + w], qkv[(n0 + u) * 3 * a.d + h * a.dh + lane], dk);
    }
    dqkv[v * 3 * a.d + a.d + h * a.dh + lane] = dk * a.scale;
    dqkv[v * 3 * a.d + 2 * a.d + h * a.dh + lane] = dv;
  }
}

// LayerNorm forward (reading R7), warp per row, two-pass statistics
__global__ void k_tr_ln_fwd(const float* __restrict__ z, const float* __restrict__ gam, const float* __restrict__ bet,
                            float eps, int64_t rows, int d, float* __restrict__ y) {
  const int64_t r = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (r >= rows) return;
  const float* zr = z + r * d;
  float s = 0.f;
  for (int c = lane; c < d; c += 32) s += zr[c];
  const float mean = warp_sum(s) / d;
  float q = 0.f;
  for (int c = lane; c < d; c += 32) q += (zr[c] - mean) * (zr[c] - mean);
  const float inv = rsqrtf(warp_sum(q) / d + eps);
  for (int c = lane; c < d; c += 32) y[r * d + c] = (zr[c] - mean) * inv * gam[c] + bet[c];
}

// LayerNorm backward: dz = inv (gx - mean(gx) - xhat mean(gx xhat)), gx = dy gamma;
// xhat written for the gamma gradient
__global__ void k_tr_ln_bwd(const float* __restrict__ z, const float* __restrict__ gam, float eps, int64_t rows, int d,
                            const float* __restrict__ dy, float* __restrict__ dz, float* __restrict__ xhat) {
  const int64_t r = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (r >= rows) return;
  const float* zr = z + r * d;
  float s = 0.f;
  for (int c = lane; c < d; c += 32) s += zr[c];
  const float mean = warp_sum(s) / d;
  float q = 0.f;
  for (int c = lane; c < d; c += 32) q += (zr[c] - mean) * (zr[c] - mean);
  const float inv = rsqrtf(warp_sum(q) / d + eps);
  float m1 = 0.f, m2 = 0.f;
  for (int c = lane; c < d; c += 32) {
    const float xh = (zr[c] - mean) * inv;
    const float gx = dy[r * d + c] * gam[c];
    xhat[r * d + c] = xh;
    m1 += gx;
    m2 += gx * xh;
  }
  m1 = warp_sum(m1) / d;
  m2 = warp_sum(m2) / d;
  for (int c = lane; c < d; c += 32) {
    const float xh = xhat[r * d + c];
    dz[r * d + c] = inv * (dy[r * d + c] * gam[c] - m1 - xh * m2);
  }
}

// out[c] = sum_r A[r][c] (* B[r][c] if B): one thread per column, rows in order
__global__ void k_tr_colsum(const float* __restrict__ A, const float* __restrict__ B, int64_t rows, int cols,
                            float* __restrict__ out) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= cols) return;
  float s = 0.f;
  for (int64_t r = 0; r < rows; ++r) s += B ? A[r * cols + c] * B[r * cols + c] : A[r * cols + c];
  out[c] = s;
}

__global__ void k_tr_relu(const float* __restrict__ x, int64_t n, float* __restrict__ y) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    y[i] = fmaxf(x[i], 0.f);
}
__global__ void k_tr_relu_bwd(const float* __restrict__ pre, int64_t n, float* __restrict__ g) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    if (!(pre[i] > 0.f)) g[i] = 0.f;
}

// readout forward (Eqn 2; head P:176, R10), block per graph, d threads
__global__ void k_tr_head_fwd(const float* __restrict__ x, const int64_t* __restrict__ node_ptr, int d, int pool_mean,
                              const float* __restrict__ H1, const float* __restrict__ c1, const float* __restrict__ H2,
                              const float* __restrict__ c2, const float* __restrict__ w_o, const float* __restrict__ c_o,
                              float* __restrict__ gv, float* __restrict__ a1, float* __restrict__ a2,
                              float* __restrict__ r1, float* __restrict__ r2, float* __restrict__ y) {
  extern __shared__ float sh[];
  float* sg = sh;
  float* sr = sh + d;
  const int g = blockIdx.x, j = threadIdx.x;
  const int64_t n0 = node_ptr[g], n1 = node_ptr[g + 1];
  float s = 0.f;
  for (int64_t v = n0; v < n1; ++v) s += x[v * d + j];
  if (pool_mean) s /= (float)(n1 - n0);
  sg[j] = s;
  gv[(int64_t)g * d + j] = s;
  __syncthreads();
  float z = c1[j];
  for (int i = 0; i < d; ++i) z = fmaf(H1[(int64_t)j * d + i], sg[i], z);
  a1[(int64_t)g * d + j] = z;
  sr[j] = fmaxf(z, 0.f);
  r1[(int64_t)g * d + j] = sr[j];
  __syncthreads();
  z = c2[j];
  for (int i = 0; i < d; ++i) z = fmaf(H2[(int64_t)j * d + i], sr[i], z);
  a2[(int64_t)g * d + j] = z;
  __syncthreads();
  sg[j] = fmaxf(z, 0.f) * w_o[j];
  r2[(int64_t)g * d + j] = fmaxf(z, 0.f);
  __syncthreads();
  if (j == 0) {
    float t = c_o[0];
    for (int i = 0; i < d; ++i) t += sg[i];
    y[g] = t;
  }
}

// MAE (Eqn 3): loss = mean |y - t|, dy = sign(y - t) / G (sign(0) = 0); one block
__global__ void k_tr_mae(const float* __restrict__ y, const float* __restrict__ t, int G, float* __restrict__ loss,
                         float* __restrict__ dy) {
  __shared__ float red[256];
  float s = 0.f;
  for (int g = threadIdx.x; g < G; g += blockDim.x) {
    const float e = y[g] - t[g];
    s += fabsf(e);
    dy[g] = (e > 0.f ? 1.f : (e < 0.f ? -1.f : 0.f)) / (float)G;
  }
  red[threadIdx.x] = s;
  __syncthreads();
  for (int o = blockDim.x / 2; o; o >>= 1) {
    if ((int)threadIdx.x < o) red[threadIdx.x] += red[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0 && loss) loss[0] = red[0] / (float)G;
}

// dz2[g][j] = dy[g] w_o[j] [a2 > 0]
__global__ void k_tr_head_bwd1(const float* __restrict__ dy, const float* __restrict__ w_o, const float* __restrict__ a2,
                               int G, int d, float* __restrict__ dz2) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= (int64_t)G * d) return;
  dz2[i] = a2[i] > 0.f ? dy[i / d] * w_o[i % d] : 0.f;
}

// dx[v][j] = dg[gid[v]][j] (/ N_g for the mean pool)
__global__ void k_tr_pool_bwd(const float* __restrict__ dg, const int32_t* __restrict__ gid,
                              const int64_t* __restrict__ node_ptr, int64_t N, int d, int pool_mean, float* __restrict__ dx) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < N * d; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = i / d;
    const int g = gid[v];
    float s = dg[(int64_t)g * d + i % d];
    if (pool_mean) s /= (float)(node_ptr[g + 1] - node_ptr[g]);
    dx[i] = s;
  }
}

__global__ void k_tr_scalar_dot(const float* __restrict__ a, const float* __restrict__ b, int n, float* __restrict__ out) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    float s = 0.f;
    for (int i = 0; i < n; ++i) s += a[i] * (b ? b[i] : 1.f);
    out[0] = s;
  }
}

__global__ void k_tr_adam(float* __restrict__ p, const float* __restrict__ g, float* __restrict__ m, float* __restrict__ v,
                          int64_t n, float lr, float b1, float b2, float eps, float bc1, float bc2s) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const float gi = g[i];
    const float mi = b1 * m[i] + (1.f - b1) * gi;
    const float vi = b2 * v[i] + (1.f - b2) * gi * gi;
    m[i] = mi;
    v[i] = vi;
    p[i] -= (lr / bc1) * mi / (sqrtf(vi) / bc2s + eps);
  }
}

// ---------------------------------------------------------------- workspace
struct TrWs {
  int32_t* gid;
  float *F, *xs, *qkv, *att, *z1, *h, *up, *z2, *u, *P, *dS;
  float *gv, *a1, *a2, *r1, *r2, *y, *dy, *dz2g, *dr1, *dg;
  float *dx, *dz, *dh, *du, *da, *dqkv, *xhat;
};
size_t carve(const predtop_train_s* tr, const predtop_dag_s* dag, void* base, TrWs* w) {
  const int64_t N = dag->desc.total_nodes, G = dag->desc.num_graphs;
  const int64_t d = tr->cfg.d_model, f = tr->cfg.d_ff, L = tr->cfg.num_layers, H = tr->cfg.num_heads;
  const int64_t PB = std::max<int64_t>(1, dag->tiles_bound) * 16384 * H;  // P floats per layer
  Carver c(base);
  TrWs t{};
  t.gid = c.take<int32_t>(N);
  t.F = c.take<float>(N * kF);
  t.xs = c.take<float>((L + 1) * N * d);
  t.qkv = c.take<float>(L * N * 3 * d);
  t.att = c.take<float>(L * N * d);
  t.z1 = c.take<float>(L * N * d);
  t.h = c.take<float>(L * N * d);
  t.up = c.take<float>(L * N * f);
  t.z2 = c.take<float>(L * N * d);
  t.u = c.take<float>(N * f);
  t.P = c.take<float>(L * PB);
  t.dS = c.take<float>(PB);
  t.gv = c.take<float>(G * d);
  t.a1 = c.take<float>(G * d);
  t.a2 = c.take<float>(G * d);
  t.r1 = c.take<float>(G * d);
  t.r2 = c.take<float>(G * d);
  t.y = c.take<float>(G);
  t.dy = c.take<float>(G);
  t.dz2g = c.take<float>(G * d);
  t.dr1 = c.take<float>(G * d);
  t.dg = c.take<float>(G * d);
  t.dx = c.take<float>(N * d);
  t.dz = c.take<float>(N * d);
  t.dh = c.take<float>(N * d);
  t.du = c.take<float>(N * f);
  t.da = c.take<float>(N * d);
  t.dqkv = c.take<float>(N * 3 * d);
  t.xhat = c.take<float>(N * d);
  if (w) *w = t;
  return c.used + 256;
}

inline unsigned blocks_for(int64_t n, int threads = 256) {
  return (unsigned)std::min<int64_t>(std::max<int64_t>(1, ceil_div(n, threads)), 148 * 32);
}

}  // namespace
}  // namespace predtop

using namespace predtop;

size_t predtop_train_state_bytes(const predtop_model_config* cfg) {
  if (!train_cfg_ok(cfg)) return 0;
  return 4 * align_up(sizeof(float) * (size_t)offsets(*cfg).total, 256);
}

predtop_status predtop_train_create(const predtop_model_config* cfg, const float* weights_host, size_t num_floats,
                                    void* device_state, size_t state_bytes, predtop_train* out) {
  if (!out || !weights_host || !device_state) { set_error("NULL argument"); return PREDTOP_ERR_INVALID_ARG; }
  *out = nullptr;
  if (!train_cfg_ok(cfg)) { set_error("unsupported training config"); return PREDTOP_ERR_UNSUPPORTED; }
  const Offs o = offsets(*cfg);
  if ((int64_t)num_floats != o.total) { set_error("weight blob has %zu floats, expected %lld", num_floats, (long long)o.total); return PREDTOP_ERR_INVALID_ARG; }
  if (state_bytes < predtop_train_state_bytes(cfg) || ((uintptr_t)device_state & 255)) {
    set_error("train state too small or misaligned");
    return PREDTOP_ERR_WORKSPACE;
  }
  auto* tr = new predtop_train_s{};
  tr->cfg = *cfg;
  tr->nparam = o.total;
  const size_t stride = align_up(sizeof(float) * (size_t)o.total, 256);
  for (int i = 0; i < 4; ++i) tr->buf[i] = reinterpret_cast<float*>((char*)device_state + i * stride);
  if (cudaGetDevice(&tr->device) != cudaSuccess ||
      cudaMemcpy(tr->buf[0], weights_host, sizeof(float) * o.total, cudaMemcpyHostToDevice) != cudaSuccess ||
      cudaMemset(tr->buf[1], 0, 3 * stride) != cudaSuccess) {
    set_error("train state upload failed: %s", cudaGetErrorString(cudaGetLastError()));
    delete tr;
    return PREDTOP_ERR_CUDA;
  }
  if (cublasCreate(&tr->blas) != CUBLAS_STATUS_SUCCESS) {
    set_error("cublasCreate failed");
    delete tr;
    return PREDTOP_ERR_CUDA;
  }
  cublasSetMathMode(tr->blas, CUBLAS_PEDANTIC_MATH);  // fp32, no TF32
  *out = tr;
  return PREDTOP_OK;
}

void predtop_train_destroy(predtop_train tr) {
  if (!tr) return;
  cublasDestroy(tr->blas);
  delete tr;
}

float* predtop_train_buffer(predtop_train tr, int32_t which) {
  return (tr && which >= 0 && which < 4) ? tr->buf[which] : nullptr;
}

size_t predtop_train_workspace(predtop_train tr, predtop_dag dag) {
  if (!tr || !dag) return 0;
  return carve(tr, dag, nullptr, nullptr);
}

predtop_status predtop_train_grad(predtop_train tr, predtop_dag dag, const float* y_true, void* workspace,
                                  size_t ws_bytes, float* loss_out, float* y_pred_out, void* cuda_stream) {
  if (!tr || !dag || !y_true || !workspace) { set_error("NULL argument"); return PREDTOP_ERR_INVALID_ARG; }
  if (((uintptr_t)workspace & 255) || ws_bytes < carve(tr, dag, nullptr, nullptr)) {
    set_error("train workspace too small or misaligned");
    return PREDTOP_ERR_WORKSPACE;
  }
  cudaStream_t st = static_cast<cudaStream_t>(cuda_stream);
  int32_t bad = -1;
  predtop_status s0 = predtop_dag_status(dag, &bad, cuda_stream);
  if (s0 != PREDTOP_OK) { set_error("training batch has an invalid graph (%d, first %d)", (int)s0, bad); return PREDTOP_ERR_INVALID_ARG; }
  TrWs w;
  carve(tr, dag, workspace, &w);
  const predtop_model_config& c = tr->cfg;
  const Offs o = offsets(c);
  const int64_t N = dag->desc.total_nodes;
  const int G = dag->desc.num_graphs;
  const int d = c.d_model, f = c.d_ff, L = c.num_layers, H = c.num_heads, dh = d / H;
  const DagDev& D = dag->d;
  const float* Wt = tr->buf[0];
  float* Gr = tr->buf[1];
  cublasHandle_t hb = tr->blas;
  PT_BLAS(cublasSetStream(hb, st));
  PT_CUDA_TRY(cudaMemsetAsync(Gr, 0, sizeof(float) * tr->nparam, st));
  AttnView av{D.node_ptr, D.row_off, D.tile_off, D.M, w.gid, H, d, dh, (float)(1.0 / std::sqrt((double)dh))};
  const unsigned warps_rows = (unsigned)ceil_div(N * H * 32, 256);
  // ---- forward
  k_tr_gid<<<std::min(G, 4096), 256, 0, st>>>(D.node_ptr, G, w.gid);
  PT_LAUNCH_CHECK();
  k_tr_features<<<blocks_for(N * kF), 256, 0, st>>>(D.feats, N, w.F);
  PT_LAUNCH_CHECK();
  PT_BLAS(gemm(hb, false, true, (int)N, d, kF, w.F, kF, Wt + o.W_in, kF, 0.f, w.xs, d));
  k_tr_embed_finish<<<blocks_for(N * d), 256, 0, st>>>(w.xs, Wt + o.b_in, D.depth, N, d);
  PT_LAUNCH_CHECK();
  for (int l = 0; l < L; ++l) {
    const auto& P = o.l[l];
    const float* x = w.xs + (int64_t)l * N * d;
    float* qkv = w.qkv + (int64_t)l * N * 3 * d;
    float* att = w.att + (int64_t)l * N * d;
    float* z1 = w.z1 + (int64_t)l * N * d;
    float* hh = w.h + (int64_t)l * N * d;
    float* up = w.up + (int64_t)l * N * f;
    float* z2 = w.z2 + (int64_t)l * N * d;
    float* Pl = w.P + (int64_t)l * std::max<int64_t>(1, dag->tiles_bound) * 16384 * H;
    k_tr_init_rows<<<blocks_for(N * 3 * d), 256, 0, st>>>(qkv, Wt + P.bqkv, nullptr, N, 3 * d);
    PT_LAUNCH_CHECK();
    PT_BLAS(gemm(hb, false, true, (int)N, 3 * d, d, x, d, Wt + P.Wqkv, d, 1.f, qkv, 3 * d));
    k_tr_attn_fwd<<<warps_rows, 256, 0, st>>>(av, N, qkv, Pl, att);
    PT_LAUNCH_CHECK();
    k_tr_init_rows<<<blocks_for(N * d), 256, 0, st>>>(z1, Wt + P.bo, x, N, d);
    PT_LAUNCH_CHECK();
    PT_BLAS(gemm(hb, false, true, (int)N, d, d, att, d, Wt + P.Wo, d, 1.f, z1, d));
    k_tr_ln_fwd<<<(unsigned)ceil_div(N * 32, 256), 256, 0, st>>>(z1, Wt + P.g1, Wt + P.be1, c.ln_eps, N, d, hh);
    PT_LAUNCH_CHECK();
    k_tr_init_rows<<<blocks_for(N * f), 256, 0, st>>>(up, Wt + P.b1, nullptr, N, f);
    PT_LAUNCH_CHECK();
    PT_BLAS(gemm(hb, false, true, (int)N, f, d, hh, d, Wt + P.W1, d, 1.f, up, f));
    k_tr_relu<<<blocks_for(N * f), 256, 0, st>>>(up, N * f, w.u);
    PT_LAUNCH_CHECK();
    k_tr_init_rows<<<blocks_for(N * d), 256, 0, st>>>(z2, Wt + P.b2, hh, N, d);
    PT_LAUNCH_CHECK();
    PT_BLAS(gemm(hb, false, true, (int)N, d, f, w.u, f, Wt + P.W2, f, 1.f, z2, d));
    k_tr_ln_fwd<<<(unsigned)ceil_div(N * 32, 256), 256, 0, st>>>(z2, Wt + P.g2, Wt + P.be2, c.ln_eps, N, d,
                                                                   w.xs + (int64_t)(l + 1) * N * d);
    PT_LAUNCH_CHECK();
  }
  const float* xL = w.xs + (int64_t)L * N * d;
  k_tr_head_fwd<<<G, d, 2 * d * sizeof(float), st>>>(xL, D.node_ptr, d, c.pool, Wt + o.H1, Wt + o.c1, Wt + o.H2,
                                                     Wt + o.c2, Wt + o.w_o, Wt + o.c_o, w.gv, w.a1, w.a2, w.r1,
                                                     w.r2, w.y);
  PT_LAUNCH_CHECK();
  k_tr_mae<<<1, 256, 0, st>>>(w.y, y_true, G, loss_out, w.dy);
  PT_LAUNCH_CHECK();
  if (y_pred_out) PT_CUDA_TRY(cudaMemcpyAsync(y_pred_out, w.y, sizeof(float) * G, cudaMemcpyDeviceToDevice, st));
  // ---- backward: head (R10) and pool (Eqn 2)
  k_tr_scalar_dot<<<1, 32, 0, st>>>(w.dy, nullptr, G, Gr + o.c_o);
  PT_LAUNCH_CHECK();
  PT_BLAS(gemm(hb, true, false, 1, d, G, w.dy, 1, w.r2, d, 0.f, Gr + o.w_o, d));  // dw_o = dy^T r2
  k_tr_head_bwd1<<<blocks_for((int64_t)G * d), 256, 0, st>>>(w.dy, Wt + o.w_o, w.a2, G, d, w.dz2g);
  PT_LAUNCH_CHECK();
  PT_BLAS(gemm(hb, true, false, d, d, G, w.dz2g, d, w.r1, d, 0.f, Gr + o.H2, d));  // dH2 = dz2^T r1
  k_tr_colsum<<<(unsigned)ceil_div(d, 128), 128, 0, st>>>(w.dz2g, nullptr, G, d, Gr + o.c2);
  PT_LAUNCH_CHECK();
  PT_BLAS(gemm(hb, false, false, G, d, d, w.dz2g, d, Wt + o.H2, d, 0.f, w.dr1, d));  // dr1 = dz2 H2
  k_tr_relu_bwd<<<blocks_for((int64_t)G * d), 256, 0, st>>>(w.a1, (int64_t)G * d, w.dr1);
  PT_LAUNCH_CHECK();
  PT_BLAS(gemm(hb, true, false, d, d, G, w.dr1, d, w.gv, d, 0.f, Gr + o.H1, d));  // dH1 = dz1^T g
  k_tr_colsum<<<(unsigned)ceil_div(d, 128), 128, 0, st>>>(w.dr1, nullptr, G, d, Gr + o.c1);
  PT_LAUNCH_CHECK();
  PT_BLAS(gemm(hb, false, false, G, d, d, w.dr1, d, Wt + o.H1, d, 0.f, w.dg, d));  // dg = dz1 H1
  k_tr_pool_bwd<<<blocks_for(N * d), 256, 0, st>>>(w.dg, w.gid, D.node_ptr, N, d, c.pool, w.dx);
  PT_LAUNCH_CHECK();
  // ---- backward: layers in reverse
  for (int l = L - 1; l >= 0; --l) {
    const auto& P = o.l[l];
    const auto& Q = o.l[l];
    const float* x = w.xs + (int64_t)l * N * d;
    const float* qkv = w.qkv + (int64_t)l * N * 3 * d;
    const float* att = w.att + (int64_t)l * N * d;
    const float* z1 = w.z1 + (int64_t)l * N * d;
    const float* hh = w.h + (int64_t)l * N * d;
    const float* up = w.up + (int64_t)l * N * f;
    const float* z2 = w.z2 + (int64_t)l * N * d;
    const float* Pl = w.P + (int64_t)l * std::max<int64_t>(1, dag->tiles_bound) * 16384 * H;
    const unsigned lnb = (unsigned)ceil_div(N * 32, 256);
    const unsigned cs = (unsigned)ceil_div(d, 128);
    // x' = LN2(z2)
    k_tr_ln_bwd<<<lnb, 256, 0, st>>>(z2, Wt + P.g2, c.ln_eps, N, d, w.dx, w.dz, w.xhat);
    PT_LAUNCH_CHECK();
    k_tr_colsum<<<cs, 128, 0, st>>>(w.dx, w.xhat, N, d, Gr + Q.g2);
    PT_LAUNCH_CHECK();
    k_tr_colsum<<<cs, 128, 0, st>>>(w.dx, nullptr, N, d, Gr + Q.be2);
    PT_LAUNCH_CHECK();
    // z2 = h + W2 u + b2
    k_tr_relu<<<blocks_for(N * f), 256, 0, st>>>(up, N * f, w.u);
    PT_LAUNCH_CHECK();
    PT_BLAS(gemm(hb, true, false, d, f, (int)N, w.dz, d, w.u, f, 0.f, Gr + Q.W2, f));  // dW2 = dz^T u
    k_tr_colsum<<<cs, 128, 0, st>>>(w.dz, nullptr, N, d, Gr + Q.b2);
    PT_LAUNCH_CHECK();
    PT_BLAS(gemm(hb, false, false, (int)N, f, d, w.dz, d, Wt + P.W2, f, 0.f, w.du, f));  // du = dz W2
    // u = ReLU(W1 h + b1)
    k_tr_relu_bwd<<<blocks_for(N * f), 256, 0, st>>>(up, N * f, w.du);
    PT_LAUNCH_CHECK();
    PT_BLAS(gemm(hb, true, false, f, d, (int)N, w.du, f, hh, d, 0.f, Gr + Q.W1, d));  // dW1 = du^T h
    k_tr_colsum<<<(unsigned)ceil_div(f, 128), 128, 0, st>>>(w.du, nullptr, N, f, Gr + Q.b1);
    PT_LAUNCH_CHECK();
    PT_CUDA_TRY(cudaMemcpyAsync(w.dh, w.dz, sizeof(float) * N * d, cudaMemcpyDeviceToDevice, st));
    PT_BLAS(gemm(hb, false, false, (int)N, d, f, w.du, f, Wt + P.W1, d, 1.f, w.dh, d));  // dh += du W1
    // h = LN1(z1)
    k_tr_ln_bwd<<<lnb, 256, 0, st>>>(z1, Wt + P.g1, c.ln_eps, N, d, w.dh, w.dz, w.xhat);
    PT_LAUNCH_CHECK();
    k_tr_colsum<<<cs, 128, 0, st>>>(w.dh, w.xhat, N, d, Gr + Q.g1);
    PT_LAUNCH_CHECK();
    k_tr_colsum<<<cs, 128, 0, st>>>(w.dh, nullptr, N, d, Gr + Q.be1);
    PT_LAUNCH_CHECK();
    // z1 = x + W_o a + b_o
    PT_BLAS(gemm(hb, true, false, d, d, (int)N, w.dz, d, att, d, 0.f, Gr + Q.Wo, d));  // dWo = dz^T a
    k_tr_colsum<<<cs, 128, 0, st>>>(w.dz, nullptr, N, d, Gr + Q.bo);
    PT_LAUNCH_CHECK();
    PT_BLAS(gemm(hb, false, false, (int)N, d, d, w.dz, d, Wt + P.Wo, d, 0.f, w.da, d));  // da = dz Wo
    // attention (Eqn 1)
    k_tr_attn_bwd_rows<<<warps_rows, 256, 0, st>>>(av, N, qkv, Pl, w.da, w.dS, w.dqkv);
    PT_LAUNCH_CHECK();
    k_tr_attn_bwd_keys<<<warps_rows, 256, 0, st>>>(av, N, qkv, Pl, w.dS, w.da, w.dqkv);
    PT_LAUNCH_CHECK();
    // qkv = W_qkv x + b_qkv; dx = dz (residual) + dqkv W_qkv
    PT_BLAS(gemm(hb, true, false, 3 * d, d, (int)N, w.dqkv, 3 * d, x, d, 0.f, Gr + Q.Wqkv, d));
    k_tr_colsum<<<(unsigned)ceil_div(3 * d, 128), 128, 0, st>>>(w.dqkv, nullptr, N, 3 * d, Gr + Q.bqkv);
    PT_LAUNCH_CHECK();
    PT_CUDA_TRY(cudaMemcpyAsync(w.dx, w.dz, sizeof(float) * N * d, cudaMemcpyDeviceToDevice, st));
    PT_BLAS(gemm(hb, false, false, (int)N, d, 3 * d, w.dqkv, 3 * d, Wt + P.Wqkv, d, 1.f, w.dx, d));
  }
  // embedding: x0 = W_in f + b_in + PE
  PT_BLAS(gemm(hb, true, false, d, kF, (int)N, w.dx, d, w.F, kF, 0.f, Gr + o.W_in, kF));
  k_tr_colsum<<<(unsigned)ceil_div(d, 128), 128, 0, st>>>(w.dx, nullptr, N, d, Gr + o.b_in);
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}

predtop_status predtop_train_adam(predtop_train tr, float lr, int32_t step, float beta1, float beta2, float eps,
                                  void* cuda_stream) {
  if (!tr) { set_error("NULL train state"); return PREDTOP_ERR_INVALID_ARG; }
  if (step < 1 || !(beta1 >= 0.f && beta1 < 1.f) || !(beta2 >= 0.f && beta2 < 1.f) || !(eps > 0.f)) {
    set_error("bad Adam arguments");
    return PREDTOP_ERR_INVALID_ARG;
  }
  const float bc1 = (float)(1.0 - std::pow((double)beta1, step));
  const float bc2s = (float)std::sqrt(1.0 - std::pow((double)beta2, step));
  k_tr_adam<<<blocks_for(tr->nparam), 256, 0, static_cast<cudaStream_t>(cuda_stream)>>>(
      tr->buf[0], tr->buf[1], tr->buf[2], tr->buf[3], tr->nparam, lr, beta1, beta2, eps, bc1, bc2s);
  PT_LAUNCH_CHECK();
  return PREDTOP_OK;
}
