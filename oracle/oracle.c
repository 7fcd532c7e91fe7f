/*
 * oracle.c -- plain CPU fp64 oracle of the PredTOP prediction path.
 * TEST INFRASTRUCTURE ONLY (see oracle.h).  Slow and obviously correct:
 * one graph at a time, textbook loops, no blocking, fusion or reordering.
 * Compile with -ffp-contract=off (no FMA contraction; Eqn 4 rounding rule R13).
 */
#include "oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------ */
/* Graph checks ("DL models are often represented as DAGs"; the stage  */
/* graph of SIV-B2).  Precedence: RANGE, then SELF_LOOP, then CYCLE.   */
/* Cycle test: iterative DFS with white/grey/black colouring.                 */
/* ------------------------------------------------------------------------ */
typedef struct {
  int* off; /* n+1 */
  int* adj; /* e   */
} orc_csr;

static orc_csr build_csr(int n, int e, const int32_t* from, const int32_t* to) {
  orc_csr g;
  g.off = (int*)calloc((size_t)n + 1, sizeof(int));
  g.adj = (int*)malloc(sizeof(int) * (size_t)(e > 0 ? e : 1));
  for (int i = 0; i < e; ++i) g.off[from[i] + 1]++;
  for (int v = 0; v < n; ++v) g.off[v + 1] += g.off[v];
  int* fill = (int*)malloc(sizeof(int) * (size_t)(n > 0 ? n : 1));
  for (int v = 0; v < n; ++v) fill[v] = g.off[v];
  for (int i = 0; i < e; ++i) g.adj[fill[from[i]]++] = to[i];
  free(fill);
  return g;
}
static void free_csr(orc_csr* g) { free(g->off); free(g->adj); }

int orc_validate(int n, int e, const int32_t* src, const int32_t* dst) {
  for (int i = 0; i < e; ++i)
    if (src[i] < 0 || src[i] >= n || dst[i] < 0 || dst[i] >= n) return ORC_RANGE;
  for (int i = 0; i < e; ++i)
    if (src[i] == dst[i]) return ORC_SELF_LOOP;
  orc_csr succ = build_csr(n, e, src, dst);
  char* colour = (char*)calloc((size_t)n + 1, 1); /* 0 white, 1 grey, 2 black */
  int* stack = (int*)malloc(sizeof(int) * ((size_t)n + 1));
  int* next = (int*)malloc(sizeof(int) * ((size_t)n + 1)); /* next successor index */
  int status = ORC_OK;
  for (int r = 0; r < n && status == ORC_OK; ++r) {
    if (colour[r]) continue;
    int sp = 0;
    stack[sp++] = r;
    colour[r] = 1;
    next[r] = succ.off[r];
    while (sp > 0 && status == ORC_OK) {
      int v = stack[sp - 1];
      if (next[v] < succ.off[v + 1]) {
        int w = succ.adj[next[v]++];
        if (colour[w] == 1) status = ORC_CYCLE;   /* back edge */
        else if (colour[w] == 0) {
          colour[w] = 1;
          next[w] = succ.off[w];
          stack[sp++] = w;
        }
      } else {
        colour[v] = 2;
        --sp;
      }
    }
  }
  free(colour); free(stack); free(next); free_csr(&succ);
  return status;
}

/* ------------------------------------------------------------------------ */
/* DAGPE depth ("using the depth of the nodes as the positional        */
/* encoding"; reading R4): depth(v) = 0 if v has no predecessor, otherwise    */
/* 1 + max_{p in pred(v)} depth(p).  Memoised recursion over predecessors,   */
/* written with an explicit stack.  Requires an acyclic graph.               */
/* ------------------------------------------------------------------------ */
void orc_depth(int n, int e, const int32_t* src, const int32_t* dst, int32_t* depth) {
  orc_csr pred = build_csr(n, e, dst, src);
  int* stack = (int*)malloc(sizeof(int) * ((size_t)n + (size_t)e + 1));
  for (int v = 0; v < n; ++v) depth[v] = -1;
  for (int r = 0; r < n; ++r) {
    if (depth[r] >= 0) continue;
    int sp = 0;
    stack[sp++] = r;
    while (sp > 0) {
      int v = stack[sp - 1];
      int ready = 1;
      for (int i = pred.off[v]; i < pred.off[v + 1]; ++i) {
        int p = pred.adj[i];
        if (depth[p] < 0) { stack[sp++] = p; ready = 0; }
      }
      if (!ready) continue;
      int best = -1; /* max over predecessors; -1 + 1 = 0 for a source */
      for (int i = pred.off[v]; i < pred.off[v + 1]; ++i)
        if (depth[pred.adj[i]] > best) best = depth[pred.adj[i]];
      depth[v] = best + 1;
      --sp;
    }
  }
  free(stack); free_csr(&pred);
}

/* ------------------------------------------------------------------------ */
/* DAGRA reachability ("a node n will attend to another node m if and  */
/* only if there exists a path from m to n or vice versa"; P:145 k = inf).   */
/* R[v] = { u != v : v reaches u by a directed path of >= 1 edge }, one      */
/* iterative DFS along successors per v.  Layout (include/predtop.h): row v  */
/* is W = 2*ceil(n/128) uint64 words, bit u%64 of word u/64; padding 0.      */
/* ------------------------------------------------------------------------ */
int orc_row_words(int n) { return 2 * ((n + 127) / 128); }

void orc_reach(int n, int e, const int32_t* src, const int32_t* dst, uint64_t* R) {
  int W = orc_row_words(n);
  memset(R, 0, sizeof(uint64_t) * (size_t)n * (size_t)W);
  orc_csr succ = build_csr(n, e, src, dst);
  char* seen = (char*)malloc((size_t)n + 1);
  int* stack = (int*)malloc(sizeof(int) * ((size_t)e + (size_t)n + 1));
  for (int v = 0; v < n; ++v) {
    memset(seen, 0, (size_t)n);
    int sp = 0;
    for (int i = succ.off[v]; i < succ.off[v + 1]; ++i) stack[sp++] = succ.adj[i];
    while (sp > 0) {
      int u = stack[--sp];
      if (seen[u]) continue;
      seen[u] = 1;
      for (int i = succ.off[u]; i < succ.off[u + 1]; ++i)
        if (!seen[succ.adj[i]]) stack[sp++] = succ.adj[i];
    }
    for (int u = 0; u < n; ++u)
      if (seen[u] && u != v) R[(size_t)v * W + (size_t)(u / 64)] |= (uint64_t)1 << (u % 64);
  }
  free(seen); free(stack); free_csr(&succ);
}

/* ------------------------------------------------------------------------ */
/* Finite-k DAGRA ("u in N_k(v)"; "the constant k ... specifies  */
/* the neighborhood range for attention calculation").       */
/* Reading R19: N_k(v) = the nodes joined to v by a directed path of at most */
/* k edges in either direction (the DAG Transformer's k-hop receptive field).*/
/* R_k[v] = { u != v : the shortest directed path v ~> u has 1..k edges },   */
/* by one breadth-first search along successors per v, stopped at depth k.   */
/* k <= 0 means k = infinity, i.e. orc_reach.                        */
/* ------------------------------------------------------------------------ */
void orc_reach_k(int n, int e, const int32_t* src, const int32_t* dst, int k, uint64_t* R) {
  if (k <= 0) { orc_reach(n, e, src, dst, R); return; }
  int W = orc_row_words(n);
  memset(R, 0, sizeof(uint64_t) * (size_t)n * (size_t)W);
  orc_csr succ = build_csr(n, e, src, dst);
  int* dist = (int*)malloc(sizeof(int) * ((size_t)n + 1));
  int* queue = (int*)malloc(sizeof(int) * ((size_t)n + 1));
  for (int v = 0; v < n; ++v) {
    for (int u = 0; u < n; ++u) dist[u] = -1;
    int head = 0, tail = 0;
    dist[v] = 0;
    queue[tail++] = v;
    while (head < tail) {
      int u = queue[head++];
      if (dist[u] == k) continue; /* do not expand past k edges */
      for (int i = succ.off[u]; i < succ.off[u + 1]; ++i) {
        int w = succ.adj[i];
        if (dist[w] < 0) { dist[w] = dist[u] + 1; queue[tail++] = w; }
      }
    }
    for (int u = 0; u < n; ++u)
      if (u != v && dist[u] >= 1 && dist[u] <= k)
        R[(size_t)v * W + (size_t)(u / 64)] |= (uint64_t)1 << (u % 64);
  }
  free(dist); free(queue); free_csr(&succ);
}

static int bit(const uint64_t* B, int W, int row, int col) {
  return (int)((B[(size_t)row * W + (size_t)(col / 64)] >> (col % 64)) & 1u);
}

/* Eqn 1 mask: M(u,v) = 0 (allowed) iff u in N_inf(v).  With     */
/* P:135 "or vice versa" the relation is symmetric (R3), and a node attends  */
/* to itself (R2): allowed(u,v) = [u == v] or R[u][v] or R[v][u].            */
void orc_mask(int n, const uint64_t* R, uint64_t* M) {
  int W = orc_row_words(n);
  memset(M, 0, sizeof(uint64_t) * (size_t)n * (size_t)W);
  for (int u = 0; u < n; ++u)
    for (int v = 0; v < n; ++v)
      if (u == v || bit(R, W, u, v) || bit(R, W, v, u))
        M[(size_t)u * W + (size_t)(v / 64)] |= (uint64_t)1 << (v % 64);
}

/* Block classes of M over 128x128 tiles (clipped to n): 0 no allowed pair,   */
/* 2 all allowed, 1 otherwise.  Returns |A| = number of allowed pairs.       */
int64_t orc_tiles(int n, const uint64_t* M, uint8_t* cls) {
  int W = orc_row_words(n);
  int T = (n + 127) / 128;
  int64_t total = 0;
  for (int qt = 0; qt < T; ++qt)
    for (int kt = 0; kt < T; ++kt) {
      int64_t cnt = 0, cells = 0;
      for (int u = qt * 128; u < n && u < qt * 128 + 128; ++u)
        for (int v = kt * 128; v < n && v < kt * 128 + 128; ++v) {
          cells++;
          cnt += bit(M, W, u, v);
        }
      if (cls) cls[qt * T + kt] = (uint8_t)(cnt == 0 ? 0 : (cnt == cells ? 2 : 1));
      total += cnt;
    }
  return total;
}

/* ------------------------------------------------------------------------ */
/* Weight blob walk (order documented in include/predtop.h).                 */
/* ------------------------------------------------------------------------ */
typedef struct {
  const float *W_in, *b_in;
  const float *H1, *c1, *H2, *c2, *w_o, *c_o;
} orc_top;
typedef struct {
  const float *Wqkv, *bqkv, *Wo, *bo, *g1, *be1, *W1, *b1, *W2, *b2, *g2, *be2;
} orc_lw;

static long layer_floats(const orc_cfg* c) {
  long d = c->d, f = c->d_ff;
  return 3 * d * d + 3 * d + d * d + d + 2 * d + f * d + f + d * f + d + 2 * d;
}

long orc_blob_floats(const orc_cfg* c) {
  long d = c->d;
  return d * ORC_F + d + (long)c->L * layer_floats(c) + 2 * (d * d + d) + d + 1;
}

static orc_lw layer_weights(const orc_cfg* c, const float* blob, int l) {
  long d = c->d, f = c->d_ff;
  const float* p = blob + d * ORC_F + d + (long)l * layer_floats(c);
  orc_lw w;
  w.Wqkv = p; p += 3 * d * d;
  w.bqkv = p; p += 3 * d;
  w.Wo = p; p += d * d;
  w.bo = p; p += d;
  w.g1 = p; p += d;
  w.be1 = p; p += d;
  w.W1 = p; p += f * d;
  w.b1 = p; p += f;
  w.W2 = p; p += d * f;
  w.b2 = p; p += d;
  w.g2 = p; p += d;
  w.be2 = p;
  return w;
}

static orc_top top_weights(const orc_cfg* c, const float* blob) {
  long d = c->d;
  orc_top t;
  t.W_in = blob;
  t.b_in = blob + d * ORC_F;
  const float* p = blob + d * ORC_F + d + (long)c->L * layer_floats(c);
  t.H1 = p; p += d * d;
  t.c1 = p; p += d;
  t.H2 = p; p += d * d;
  t.c2 = p; p += d;
  t.w_o = p; p += d;
  t.c_o = p;
  return t;
}

/* y[r][o] = b[o] + sum_i W[o][i] x[r][i]   (PyTorch Linear, W is [out][in]) */
static void linear(int rows, int in, int out, const double* x, const float* W, const float* b,
                   double* y) {
  for (int r = 0; r < rows; ++r)
    for (int o = 0; o < out; ++o) {
      double s = b ? (double)b[o] : 0.0;
      for (int i = 0; i < in; ++i) s += (double)W[(size_t)o * in + i] * x[(size_t)r * in + i];
      y[(size_t)r * out + o] = s;
    }
}

/* LayerNorm over the last dim, biased variance, affine (R7: eps from cfg). */
static void layer_norm(int rows, int d, const double* z, const float* g, const float* b,
                       double eps, double* y) {
  for (int r = 0; r < rows; ++r) {
    const double* zr = z + (size_t)r * d;
    double mean = 0.0;
    for (int i = 0; i < d; ++i) mean += zr[i];
    mean /= d;
    double var = 0.0;
    for (int i = 0; i < d; ++i) var += (zr[i] - mean) * (zr[i] - mean);
    var /= d;
    double inv = 1.0 / sqrt(var + eps);
    for (int i = 0; i < d; ++i) y[(size_t)r * d + i] = (zr[i] - mean) * inv * (double)g[i] + (double)b[i];
  }
}

/* ------------------------------------------------------------------------ */
/* Node features, Table I + log scaling, reading R9:     */
/* f = [onehot(op) 64 | ln(1+dim_j) j<4 | onehot(dtype) 8 | onehot(kind) 4]. */
/* Out-of-vocabulary ids give an all-zero one-hot block.                      */
/* ------------------------------------------------------------------------ */
void orc_features(int n, const orc_feat* feats, double* f) {
  memset(f, 0, sizeof(double) * (size_t)n * ORC_F);
  for (int v = 0; v < n; ++v) {
    double* fv = f + (size_t)v * ORC_F;
    if (feats[v].op < ORC_NUM_OPS) fv[feats[v].op] = 1.0;
    for (int j = 0; j < ORC_NUM_DIMS; ++j) fv[ORC_NUM_OPS + j] = log1p((double)feats[v].dims[j]);
    if (feats[v].dtype < ORC_NUM_DTYPES) fv[ORC_NUM_OPS + ORC_NUM_DIMS + feats[v].dtype] = 1.0;
    if (feats[v].kind < ORC_NUM_KINDS)
      fv[ORC_NUM_OPS + ORC_NUM_DIMS + ORC_NUM_DTYPES + feats[v].kind] = 1.0;
  }
}

/* x0 = W_in f(v) + b_in + PE(depth(v)).  PE is the sinusoidal encoding of   */
/* [34] applied to the depth (reading R5):                            */
/*   PE[2i] = sin(depth * w_i), PE[2i+1] = cos(depth * w_i),                 */
/*   w_i = 10000^(-2i/d).                                                    */
void orc_embed(const orc_cfg* c, const float* blob, int n, const orc_feat* feats,
               const int32_t* depth, double* x0) {
  int d = c->d;
  orc_top t = top_weights(c, blob);
  double* f = (double*)malloc(sizeof(double) * (size_t)n * ORC_F);
  orc_features(n, feats, f);
  linear(n, ORC_F, d, f, t.W_in, t.b_in, x0);
  for (int v = 0; v < n; ++v)
    for (int i = 0; 2 * i < d; ++i) {
      double w = pow(10000.0, -(2.0 * i) / d);
      x0[(size_t)v * d + 2 * i] += sin(depth[v] * w);
      if (2 * i + 1 < d) x0[(size_t)v * d + 2 * i + 1] += cos(depth[v] * w);
    }
  free(f);
}

/* ------------------------------------------------------------------------ */
/* Eqn 1 with V (reading R1): per head h,                         */
/*   O_h = softmax(Q_h K_h^T / sqrt(d_h) + M) V_h,  M in {0, -inf}.          */
/* Softmax is the plain two-pass form over the allowed set (max, exp, sum).  */
/* Output: concat_h O_h, [n][d].                                             */
/* ------------------------------------------------------------------------ */
/* q|k|v rows [r0, r1) of layer `layer`: qkv[u] = W_qkv x[u] + b_qkv.       */
void orc_qkv_rows(const orc_cfg* c, const float* blob, int layer, int r0, int r1, const double* x,
                  double* qkv) {
  int d = c->d;
  orc_lw w = layer_weights(c, blob, layer);
  linear(r1 - r0, d, 3 * d, x + (size_t)r0 * d, w.Wqkv, w.bqkv, qkv + (size_t)r0 * 3 * d);
}

/* Attention output rows u in [r0, r1) from the full q|k|v matrix [n][3d].   */
void orc_attention_rows(const orc_cfg* c, int n, const uint64_t* M, const double* qkv, int r0, int r1,
                        double* concat_out) {
  int d = c->d, H = c->H, dh = c->d / c->H;
  int W = orc_row_words(n);
  double* s = (double*)malloc(sizeof(double) * (size_t)n);
  double scale = 1.0 / sqrt((double)dh);
  for (int h = 0; h < H; ++h)
    for (int u = r0; u < r1; ++u) {
      const double* q = qkv + (size_t)u * 3 * d + h * dh;
      double mx = -INFINITY;
      for (int v = 0; v < n; ++v) {
        if (!bit(M, W, u, v)) continue;
        const double* k = qkv + (size_t)v * 3 * d + d + h * dh;
        double acc = 0.0;
        for (int j = 0; j < dh; ++j) acc += q[j] * k[j];
        s[v] = acc * scale;
        if (s[v] > mx) mx = s[v];
      }
      double sum = 0.0;
      for (int v = 0; v < n; ++v)
        if (bit(M, W, u, v)) { s[v] = exp(s[v] - mx); sum += s[v]; }
      double* o = concat_out + (size_t)u * d + h * dh;
      for (int j = 0; j < dh; ++j) o[j] = 0.0;
      for (int v = 0; v < n; ++v) {
        if (!bit(M, W, u, v)) continue;
        const double* vv = qkv + (size_t)v * 3 * d + 2 * d + h * dh;
        double p = s[v] / sum;
        for (int j = 0; j < dh; ++j) o[j] += p * vv[j];
      }
    }
  free(s);
}

void orc_attention(const orc_cfg* c, const float* blob, int layer, int n, const uint64_t* M,
                   const double* x, double* concat_out) {
  double* qkv = (double*)malloc(sizeof(double) * (size_t)n * 3 * c->d);
  orc_qkv_rows(c, blob, layer, 0, n, x, qkv);
  orc_attention_rows(c, n, M, qkv, 0, n, concat_out);
  free(qkv);
}

/* DAG Transformer layer (Fig. 4; reading R6, post-LN encoder  */
/* layer of [34] with ReLU FFN):                                             */
/*   h = LN1(x + W_o a + b_o),  x' = LN2(h + W_2 ReLU(W_1 h + b_1) + b_2).   */
/* orc_layer_post_rows: everything after the attention, rows [r0, r1) of the */
/* full [n][d] arrays a (attention output), x_in and x_out (row-wise ops).   */
void orc_layer_post_rows(const orc_cfg* c, const float* blob, int layer, int r0, int r1, const double* a_full,
                         const double* x_in_full, double* x_out_full) {
  int d = c->d, f = c->d_ff, n = r1 - r0;
  orc_lw w = layer_weights(c, blob, layer);
  const double* a = a_full + (size_t)r0 * d;
  const double* x_in = x_in_full + (size_t)r0 * d;
  double* x_out = x_out_full + (size_t)r0 * d;
  double* z = (double*)malloc(sizeof(double) * (size_t)n * d);
  double* h = (double*)malloc(sizeof(double) * (size_t)n * d);
  double* u = (double*)malloc(sizeof(double) * (size_t)n * f);
  linear(n, d, d, a, w.Wo, w.bo, z);
  for (long i = 0; i < (long)n * d; ++i) z[i] += x_in[i];
  layer_norm(n, d, z, w.g1, w.be1, c->ln_eps, h);
  linear(n, d, f, h, w.W1, w.b1, u);
  for (long i = 0; i < (long)n * f; ++i) u[i] = u[i] > 0.0 ? u[i] : 0.0;
  linear(n, f, d, u, w.W2, w.b2, z);
  for (long i = 0; i < (long)n * d; ++i) z[i] += h[i];
  layer_norm(n, d, z, w.g2, w.be2, c->ln_eps, x_out);
  free(z); free(h); free(u);
}

void orc_layer(const orc_cfg* c, const float* blob, int layer, int n, const uint64_t* M,
               const double* x_in, double* x_out) {
  double* a = (double*)malloc(sizeof(double) * (size_t)n * c->d);
  orc_attention(c, blob, layer, n, M, x_in, a);
  orc_layer_post_rows(c, blob, layer, 0, n, a, x_in, x_out);
  free(a);
}

/* Readout: global add pool, Eqn 2: x_i = sum_n x_n^i (mean if the   */
/* R11 flag is set), then "linear layers each with ReLU activation, and      */
/* finally ... the output layer" (reading R10: two hidden layers of   */
/* width d, output Linear(d -> 1), no output activation).                     */
double orc_readout(const orc_cfg* c, const float* blob, int n, const double* x) {
  int d = c->d;
  orc_top t = top_weights(c, blob);
  double* g = (double*)calloc((size_t)d, sizeof(double));
  double* z1 = (double*)malloc(sizeof(double) * (size_t)d);
  double* z2 = (double*)malloc(sizeof(double) * (size_t)d);
  for (int v = 0; v < n; ++v)
    for (int j = 0; j < d; ++j) g[j] += x[(size_t)v * d + j];
  if (c->pool == 1)
    for (int j = 0; j < d; ++j) g[j] /= n;
  linear(1, d, d, g, t.H1, t.c1, z1);
  for (int j = 0; j < d; ++j) z1[j] = z1[j] > 0.0 ? z1[j] : 0.0;
  linear(1, d, d, z1, t.H2, t.c2, z2);
  for (int j = 0; j < d; ++j) z2[j] = z2[j] > 0.0 ? z2[j] : 0.0;
  double y;
  linear(1, d, 1, z2, t.w_o, t.c_o, &y);
  free(g); free(z1); free(z2);
  return y;
}

/* Whole black-box stage predictor for one stage graph.          */
/* taps (nullable): (L+1) x n x d doubles: x0, then x after each layer.      */
/* Returns the validation status; y = NaN for an invalid graph.              */
int orc_forward(const orc_cfg* c, const float* blob, int n, int e, const int32_t* src,
                const int32_t* dst, const orc_feat* feats, double* y, double* taps) {
  return orc_forward_k(c, blob, n, e, src, dst, feats, 0, y, taps);
}

/* The same forward pass with the k-hop mask M = R_k | R_k^T | I (P:142,     */
/* P:145; R19).  k <= 0 is k = infinity.                                     */
int orc_forward_k(const orc_cfg* c, const float* blob, int n, int e, const int32_t* src,
                  const int32_t* dst, const orc_feat* feats, int k, double* y, double* taps) {
  int st = orc_validate(n, e, src, dst);
  if (st != ORC_OK) { *y = NAN; return st; }
  int d = c->d, W = orc_row_words(n);
  int32_t* depth = (int32_t*)malloc(sizeof(int32_t) * (size_t)n);
  uint64_t* R = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)n * W);
  uint64_t* M = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)n * W);
  double* x = (double*)malloc(sizeof(double) * (size_t)n * d);
  double* x2 = (double*)malloc(sizeof(double) * (size_t)n * d);
  orc_depth(n, e, src, dst, depth);
  orc_reach_k(n, e, src, dst, k, R);
  orc_mask(n, R, M);
  orc_embed(c, blob, n, feats, depth, x);
  if (taps) memcpy(taps, x, sizeof(double) * (size_t)n * d);
  for (int l = 0; l < c->L; ++l) {
    orc_layer(c, blob, l, n, M, x, x2);
    double* tmp = x; x = x2; x2 = tmp;
    if (taps) memcpy(taps + (size_t)(l + 1) * n * d, x, sizeof(double) * (size_t)n * d);
  }
  *y = orc_readout(c, blob, n, x);
  free(depth); free(R); free(M); free(x); free(x2);
  return ORC_OK;
}

/* ------------------------------------------------------------------------ */
/* White-box pipeline model, Eqn 4 (definitions):              */
/*   T = sum_{i=1..S} t_i + (B - 1) * max_j t_j                              */
/* Reading R13 (canonical fp64 order): sort the plan's fp32 latencies        */
/* ascending, sum them in fp64 left to right, m = max, T = sum + (B-1)*m.    */
/* Invalid plan (S < 1, S > 64, B < 1, stage index out of range) -> NaN.     */
/* ------------------------------------------------------------------------ */
void orc_plan_T(int64_t P, const int64_t* plan_ptr, const int32_t* plan_stage,
                const int32_t* B, const float* t, int64_t num_stages, double* T) {
  float buf[64];
  for (int64_t p = 0; p < P; ++p) {
    int64_t S = plan_ptr[p + 1] - plan_ptr[p];
    int ok = S >= 1 && S <= 64 && B[p] >= 1;
    for (int64_t i = 0; ok && i < S; ++i) {
      int32_t s = plan_stage[plan_ptr[p] + i];
      if (s < 0 || s >= num_stages) ok = 0;
    }
    if (!ok) { T[p] = NAN; continue; }
    for (int64_t i = 0; i < S; ++i) buf[i] = t[plan_stage[plan_ptr[p] + i]];
    for (int64_t i = 1; i < S; ++i) { /* insertion sort, ascending */
      float key = buf[i];
      int64_t j = i - 1;
      while (j >= 0 && buf[j] > key) { buf[j + 1] = buf[j]; --j; }
      buf[j + 1] = key;
    }
    double sum = 0.0;
    for (int64_t i = 0; i < S; ++i) sum += (double)buf[i];
    double m = (double)buf[S - 1];
    double prod = (double)(B[p] - 1) * m;
    T[p] = sum + prod;
  }
}

/* argmin by (T, index) (R13); NaN never chosen; all NaN -> -1. */
int64_t orc_argmin(int64_t n, const double* T) {
  int64_t best = -1;
  for (int64_t i = 0; i < n; ++i) {
    if (isnan(T[i])) continue;
    if (best < 0 || T[i] < T[best]) best = i;
  }
  return best;
}

/* ------------------------------------------------------------------------ */
/* Inter-stage plan search over a shared stage table.       */
/* Alpa's inter-operator optimizer picks the pipeline plan with the   */
/* 1F1B model; it iterates through all possible stages and        */
/* submeshes; PredTOP predicts every stage on every mesh and applies  */
/* the pipeline model (Eqn 4).  Plain definition (reading R20): a plan       */
/* slices the L layers into S >= 1 contiguous stages [a_s, b_s] and gives    */
/* each a choice c_s (a mesh / intra-op configuration, Tables II-III) using  */
/* dev[c_s] devices, with sum_s dev[c_s] == D (the whole cluster) and every  */
/* t[a_s][b_s][c_s] feasible (finite, >= 0).  T(plan) = Eqn 4 over its S     */
/* stage latencies (orc_plan_T, R13).  The optimum is the minimum over ALL   */
/* plans, found here by exhaustive enumeration (no DP); ties keep the first  */
/* plan in the enumeration order (stage ends ascending, then choices         */
/* ascending).  Table layout: t[(i*L + j)*K + c], entries with i > j unused. */
/* Returns T* (+inf when no plan is feasible, S_out = 0).                    */
/* ------------------------------------------------------------------------ */
typedef struct {
  int L, K, D, B;
  const int32_t* dev;
  const float* t;
  int S;
  int32_t end[64], choice[64];
  double best;
  int best_S;
  int32_t best_end[64], best_choice[64];
} orc_search;

static void search_rec(orc_search* s, int k, int d) {
  if (k == s->L) {
    if (d != 0 || s->S == 0) return;
    int64_t ptr[2] = {0, s->S};
    int32_t idx[64];
    int a = 0;
    for (int i = 0; i < s->S; ++i) {
      idx[i] = (int32_t)(((int64_t)a * s->L + s->end[i]) * s->K + s->choice[i]);
      a = s->end[i] + 1;
    }
    int32_t B = s->B;
    double T;
    orc_plan_T(1, ptr, idx, &B, s->t, (int64_t)s->L * s->L * s->K, &T);
    if (T < s->best) {
      s->best = T;
      s->best_S = s->S;
      for (int i = 0; i < s->S; ++i) { s->best_end[i] = s->end[i]; s->best_choice[i] = s->choice[i]; }
    }
    return;
  }
  if (d <= 0 || s->S >= 64) return;
  for (int j = k; j < s->L; ++j)
    for (int c = 0; c < s->K; ++c) {
      float v = s->t[((int64_t)k * s->L + j) * s->K + c];
      if (!(isfinite(v) && v >= 0.0f) || s->dev[c] > d) continue;
      s->end[s->S] = j;
      s->choice[s->S] = c;
      s->S++;
      search_rec(s, j + 1, d - s->dev[c]);
      s->S--;
    }
}

double orc_plan_search(int L, int K, const int32_t* dev, int D, const float* t, int B,
                       int32_t* S_out, int32_t* stage_end, int32_t* stage_choice) {
  orc_search s;
  memset(&s, 0, sizeof(s));
  s.L = L; s.K = K; s.D = D; s.B = B; s.dev = dev; s.t = t;
  s.best = INFINITY;
  for (int c = 0; c < K; ++c)
    if (dev[c] < 1) { *S_out = 0; return NAN; }
  if (L >= 1 && L <= 64 && B >= 1) search_rec(&s, 0, D);
  *S_out = s.best_S;
  for (int i = 0; i < s.best_S; ++i) { stage_end[i] = s.best_end[i]; stage_choice[i] = s.best_choice[i]; }
  return s.best;
}

/* ------------------------------------------------------------------------ */
/* Graph pruning (SIV-B4): "operations whose effects can be      */
/* stored in the graph even after removing them ... such as reshape and     */
/* convert_element_type ... We remove these redundant operators".  Reading  */
/* R21: an OPERATOR node whose op id is in `ops` is removed; every other    */
/* node is kept, renumbered in its original order with its record unchanged;*/
/* kept u gets an edge to kept w iff the raw graph has a path u -> ... -> w */
/* of >= 1 edge whose interior nodes are all removed (the removed node's    */
/* inputs are spliced to its consumers).  Output edges are unique and       */
/* sorted by (src, dst).  Plain per-node DFS through removed nodes.         */
/* Returns ORC_OK or the validation status of the raw graph (outputs then   */
/* untouched).  out_src/out_dst must hold the result (at most nk*nk).       */
/* ------------------------------------------------------------------------ */
int orc_prune(int n, int e, const int32_t* src, const int32_t* dst, const orc_feat* feats,
              const uint16_t* ops, int n_ops, int32_t* nk_out, int32_t* out_src, int32_t* out_dst,
              int64_t* ne_out, orc_feat* out_feats) {
  int st = orc_validate(n, e, src, dst);
  if (st != ORC_OK) return st;
  char* removed = (char*)calloc((size_t)n + 1, 1);
  int* newid = (int*)malloc(sizeof(int) * ((size_t)n + 1));
  int nk = 0;
  for (int v = 0; v < n; ++v) {
    int hit = 0;
    for (int i = 0; i < n_ops; ++i) hit |= feats[v].op == ops[i];
    removed[v] = (char)(hit && feats[v].kind == 2 /* operator */);
    newid[v] = removed[v] ? -1 : nk;
    if (!removed[v]) out_feats[nk++] = feats[v];
  }
  orc_csr succ = build_csr(n, e, src, dst);
  char* seen = (char*)malloc((size_t)n + 1);
  char* target = (char*)malloc((size_t)n + 1);
  int* stack = (int*)malloc(sizeof(int) * ((size_t)e + (size_t)n + 1));
  int64_t ne = 0;
  for (int u = 0; u < n; ++u) {
    if (removed[u]) continue;
    memset(seen, 0, (size_t)n);
    memset(target, 0, (size_t)n);
    int sp = 0;
    for (int i = succ.off[u]; i < succ.off[u + 1]; ++i) stack[sp++] = succ.adj[i];
    while (sp > 0) {
      int w = stack[--sp];
      if (!removed[w]) { target[w] = 1; continue; } /* a kept node ends the path */
      if (seen[w]) continue;
      seen[w] = 1;
      for (int i = succ.off[w]; i < succ.off[w + 1]; ++i) stack[sp++] = succ.adj[i];
    }
    for (int w = 0; w < n; ++w) /* ascending kept ids = ascending new ids */
      if (target[w]) { out_src[ne] = newid[u]; out_dst[ne] = newid[w]; ++ne; }
  }
  *nk_out = nk;
  *ne_out = ne;
  free(removed); free(newid); free(seen); free(target); free(stack); free_csr(&succ);
  return ORC_OK;
}

/* ======================================================================== */
/* Training: gradient of the predicted    */
/* latency of ONE stage graph with respect to every weight of the blob,      */
/* written as the plain reverse of the forward steps above (same order,      */
/* same readings), fp64.  The MAE loss of Eqn 3 and Adam / cosine LR */
/* are composed by the caller (oracle/__init__.py).                  */
/* ======================================================================== */

/* Gradient blob views: the same float order as the weight blob. */
typedef struct {
  double *Wqkv, *bqkv, *Wo, *bo, *g1, *be1, *W1, *b1, *W2, *b2, *g2, *be2;
} orc_glw;
typedef struct {
  double *W_in, *b_in, *H1, *c1, *H2, *c2, *w_o, *c_o;
} orc_gtop;

static orc_glw grad_layer(const orc_cfg* c, double* g, int l) {
  long d = c->d, f = c->d_ff;
  double* p = g + d * ORC_F + d + (long)l * layer_floats(c);
  orc_glw w;
  w.Wqkv = p; p += 3 * d * d;
  w.bqkv = p; p += 3 * d;
  w.Wo = p; p += d * d;
  w.bo = p; p += d;
  w.g1 = p; p += d;
  w.be1 = p; p += d;
  w.W1 = p; p += f * d;
  w.b1 = p; p += f;
  w.W2 = p; p += d * f;
  w.b2 = p; p += d;
  w.g2 = p; p += d;
  w.be2 = p;
  return w;
}
static orc_gtop grad_top(const orc_cfg* c, double* g) {
  long d = c->d;
  orc_gtop t;
  t.W_in = g;
  t.b_in = g + d * ORC_F;
  double* p = g + d * ORC_F + d + (long)c->L * layer_floats(c);
  t.H1 = p; p += d * d;
  t.c1 = p; p += d;
  t.H2 = p; p += d * d;
  t.c2 = p; p += d;
  t.w_o = p; p += d;
  t.c_o = p;
  return t;
}

/* Reverse of linear(): y[r][o] = b[o] + sum_i W[o][i] x[r][i].
 * dW[o][i] += sum_r dy[r][o] x[r][i];  db[o] += sum_r dy[r][o];
 * dx[r][i] += sum_o dy[r][o] W[o][i]   (dx nullable). */
static void linear_back(int rows, int in, int out, const double* x, const float* W, const double* dy,
                        double* dW, double* db, double* dx) {
  for (int r = 0; r < rows; ++r)
    for (int o = 0; o < out; ++o) {
      double g = dy[(size_t)r * out + o];
      if (db) db[o] += g;
      for (int i = 0; i < in; ++i) {
        dW[(size_t)o * in + i] += g * x[(size_t)r * in + i];
        if (dx) dx[(size_t)r * in + i] += g * (double)W[(size_t)o * in + i];
      }
    }
}

/* Reverse of layer_norm(): y = xhat * g + b, xhat = (z - mean) * inv.
 * dg += sum_r dy*xhat; db += sum_r dy; with gx = dy*g:
 * dz = inv * (gx - mean(gx) - xhat * mean(gx * xhat))   (dz overwritten). */
static void layer_norm_back(int rows, int d, const double* z, const float* g, double eps, const double* dy,
                            double* dg, double* db, double* dz) {
  double* xh = (double*)malloc(sizeof(double) * (size_t)d);
  double* gx = (double*)malloc(sizeof(double) * (size_t)d);
  for (int r = 0; r < rows; ++r) {
    const double* zr = z + (size_t)r * d;
    const double* dyr = dy + (size_t)r * d;
    double mean = 0.0;
    for (int i = 0; i < d; ++i) mean += zr[i];
    mean /= d;
    double var = 0.0;
    for (int i = 0; i < d; ++i) var += (zr[i] - mean) * (zr[i] - mean);
    var /= d;
    double inv = 1.0 / sqrt(var + eps);
    double m1 = 0.0, m2 = 0.0;
    for (int i = 0; i < d; ++i) {
      xh[i] = (zr[i] - mean) * inv;
      gx[i] = dyr[i] * (double)g[i];
      dg[i] += dyr[i] * xh[i];
      db[i] += dyr[i];
      m1 += gx[i];
      m2 += gx[i] * xh[i];
    }
    m1 /= d;
    m2 /= d;
    for (int i = 0; i < d; ++i) dz[(size_t)r * d + i] = inv * (gx[i] - m1 - xh[i] * m2);
  }
  free(xh);
  free(gx);
}

/* Reverse of orc_attention_rows over all rows (per head h, Eqn 1):
 *   S = Q K^T / sqrt(d_h) on allowed pairs, P = softmax_row(S), O = P V.
 *   dV = P^T dO;  dP = dO V^T;  dS = P * (dP - rowsum(dP * P));
 *   dQ = dS K / sqrt(d_h);  dK = dS^T Q / sqrt(d_h).
 * dqkv [n][3d] accumulates. */
static void attention_back(const orc_cfg* c, int n, const uint64_t* M, const double* qkv, const double* dO,
                           double* dqkv) {
  int d = c->d, H = c->H, dh = c->d / c->H;
  int W = orc_row_words(n);
  double scale = 1.0 / sqrt((double)dh);
  double* P = (double*)malloc(sizeof(double) * (size_t)n);
  double* dP = (double*)malloc(sizeof(double) * (size_t)n);
  for (int h = 0; h < H; ++h)
    for (int u = 0; u < n; ++u) {
      const double* q = qkv + (size_t)u * 3 * d + h * dh;
      double mx = -INFINITY;
      for (int v = 0; v < n; ++v) {
        P[v] = 0.0;
        if (!bit(M, W, u, v)) continue;
        const double* k = qkv + (size_t)v * 3 * d + d + h * dh;
        double acc = 0.0;
        for (int j = 0; j < dh; ++j) acc += q[j] * k[j];
        P[v] = acc * scale;
        if (P[v] > mx) mx = P[v];
      }
      double sum = 0.0;
      for (int v = 0; v < n; ++v)
        if (bit(M, W, u, v)) { P[v] = exp(P[v] - mx); sum += P[v]; }
      for (int v = 0; v < n; ++v) P[v] /= sum;
      const double* dou = dO + (size_t)u * d + h * dh;
      double rs = 0.0;
      for (int v = 0; v < n; ++v) {
        dP[v] = 0.0;
        if (!bit(M, W, u, v)) continue;
        const double* vv = qkv + (size_t)v * 3 * d + 2 * d + h * dh;
        double acc = 0.0;
        for (int j = 0; j < dh; ++j) acc += dou[j] * vv[j];
        dP[v] = acc;
        rs += acc * P[v];
        double* dvv = dqkv + (size_t)v * 3 * d + 2 * d + h * dh;
        for (int j = 0; j < dh; ++j) dvv[j] += P[v] * dou[j];
      }
      double* dq = dqkv + (size_t)u * 3 * d + h * dh;
      for (int v = 0; v < n; ++v) {
        if (!bit(M, W, u, v)) continue;
        double ds = P[v] * (dP[v] - rs) * scale;
        const double* k = qkv + (size_t)v * 3 * d + d + h * dh;
        double* dk = dqkv + (size_t)v * 3 * d + d + h * dh;
        for (int j = 0; j < dh; ++j) {
          dq[j] += ds * k[j];
          dk[j] += ds * q[j];
        }
      }
    }
  free(P);
  free(dP);
}

/* Latency y of one graph (as orc_forward) and grad += dy * dy/dtheta for  */
/* every weight of the blob (grad: orc_blob_floats doubles, accumulated). */
int orc_grad(const orc_cfg* c, const float* blob, int n, int e, const int32_t* src, const int32_t* dst,
             const orc_feat* feats, double dy, double* y, double* grad) {
  int st = orc_validate(n, e, src, dst);
  if (st != ORC_OK) { *y = NAN; return st; }
  int d = c->d, f = c->d_ff, L = c->L, W = orc_row_words(n);
  size_t nd = (size_t)n * d;
  int32_t* depth = (int32_t*)malloc(sizeof(int32_t) * (size_t)n);
  uint64_t* R = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)n * W);
  uint64_t* Mk = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)n * W);
  orc_depth(n, e, src, dst, depth);
  orc_reach(n, e, src, dst, R);
  orc_mask(n, R, Mk);
  /* ---- forward with every intermediate kept */
  double* F = (double*)malloc(sizeof(double) * (size_t)n * ORC_F);
  orc_features(n, feats, F);
  double* xs = (double*)malloc(sizeof(double) * nd * (L + 1));     /* layer inputs / outputs */
  double* qkv = (double*)malloc(sizeof(double) * nd * 3 * L);
  double* att = (double*)malloc(sizeof(double) * nd * L);
  double* z1 = (double*)malloc(sizeof(double) * nd * L);
  double* hh = (double*)malloc(sizeof(double) * nd * L);
  double* up = (double*)malloc(sizeof(double) * (size_t)n * f * L); /* pre-ReLU */
  double* uu = (double*)malloc(sizeof(double) * (size_t)n * f * L);
  double* z2 = (double*)malloc(sizeof(double) * nd * L);
  orc_embed(c, blob, n, feats, depth, xs);
  for (int l = 0; l < L; ++l) {
    orc_lw w = layer_weights(c, blob, l);
    const double* x = xs + nd * l;
    double* q = qkv + nd * 3 * l;
    linear(n, d, 3 * d, x, w.Wqkv, w.bqkv, q);
    orc_attention_rows(c, n, Mk, q, 0, n, att + nd * l);
    linear(n, d, d, att + nd * l, w.Wo, w.bo, z1 + nd * l);
    for (size_t i = 0; i < nd; ++i) z1[nd * l + i] += x[i];
    layer_norm(n, d, z1 + nd * l, w.g1, w.be1, c->ln_eps, hh + nd * l);
    linear(n, d, f, hh + nd * l, w.W1, w.b1, up + (size_t)n * f * l);
    for (size_t i = 0; i < (size_t)n * f; ++i) {
      double v = up[(size_t)n * f * l + i];
      uu[(size_t)n * f * l + i] = v > 0.0 ? v : 0.0;
    }
    linear(n, f, d, uu + (size_t)n * f * l, w.W2, w.b2, z2 + nd * l);
    for (size_t i = 0; i < nd; ++i) z2[nd * l + i] += hh[nd * l + i];
    layer_norm(n, d, z2 + nd * l, w.g2, w.be2, c->ln_eps, xs + nd * (l + 1));
  }
  /* readout forward (orc_readout, intermediates kept) */
  orc_top t = top_weights(c, blob);
  const double* xL = xs + nd * L;
  double* g = (double*)calloc((size_t)d, sizeof(double));
  double* a1 = (double*)malloc(sizeof(double) * (size_t)d);
  double* a2 = (double*)malloc(sizeof(double) * (size_t)d);
  double* r1 = (double*)malloc(sizeof(double) * (size_t)d);
  double* r2 = (double*)malloc(sizeof(double) * (size_t)d);
  for (int v = 0; v < n; ++v)
    for (int j = 0; j < d; ++j) g[j] += xL[(size_t)v * d + j];
  if (c->pool == 1)
    for (int j = 0; j < d; ++j) g[j] /= n;
  linear(1, d, d, g, t.H1, t.c1, a1);
  for (int j = 0; j < d; ++j) r1[j] = a1[j] > 0.0 ? a1[j] : 0.0;
  linear(1, d, d, r1, t.H2, t.c2, a2);
  for (int j = 0; j < d; ++j) r2[j] = a2[j] > 0.0 ? a2[j] : 0.0;
  linear(1, d, 1, r2, t.w_o, t.c_o, y);
  /* ---- backward */
  orc_gtop gt = grad_top(c, grad);
  double* dr2 = (double*)calloc((size_t)d, sizeof(double));
  double* dr1 = (double*)calloc((size_t)d, sizeof(double));
  double* dg = (double*)calloc((size_t)d, sizeof(double));
  double dyv = dy;
  linear_back(1, d, 1, r2, t.w_o, &dyv, gt.w_o, gt.c_o, dr2);
  for (int j = 0; j < d; ++j) dr2[j] = a2[j] > 0.0 ? dr2[j] : 0.0;
  linear_back(1, d, d, r1, t.H2, dr2, gt.H2, gt.c2, dr1);
  for (int j = 0; j < d; ++j) dr1[j] = a1[j] > 0.0 ? dr1[j] : 0.0;
  linear_back(1, d, d, g, t.H1, dr1, gt.H1, gt.c1, dg);
  double* dx = (double*)malloc(sizeof(double) * nd);
  for (int v = 0; v < n; ++v)
    for (int j = 0; j < d; ++j) dx[(size_t)v * d + j] = c->pool == 1 ? dg[j] / n : dg[j];
  double* dz = (double*)malloc(sizeof(double) * nd);
  double* dh = (double*)malloc(sizeof(double) * nd);
  double* du = (double*)malloc(sizeof(double) * (size_t)n * f);
  double* da = (double*)malloc(sizeof(double) * nd);
  double* dq = (double*)malloc(sizeof(double) * nd * 3);
  for (int l = L - 1; l >= 0; --l) {
    orc_lw w = layer_weights(c, blob, l);
    orc_glw gw = grad_layer(c, grad, l);
    /* x' = LN2(z2) */
    layer_norm_back(n, d, z2 + nd * l, w.g2, c->ln_eps, dx, gw.g2, gw.be2, dz);
    /* z2 = h + W2 u + b2 */
    memcpy(dh, dz, sizeof(double) * nd);
    memset(du, 0, sizeof(double) * (size_t)n * f);
    linear_back(n, f, d, uu + (size_t)n * f * l, w.W2, dz, gw.W2, gw.b2, du);
    /* u = ReLU(W1 h + b1) */
    for (size_t i = 0; i < (size_t)n * f; ++i)
      if (!(up[(size_t)n * f * l + i] > 0.0)) du[i] = 0.0;
    linear_back(n, d, f, hh + nd * l, w.W1, du, gw.W1, gw.b1, dh);
    /* h = LN1(z1) */
    layer_norm_back(n, d, z1 + nd * l, w.g1, c->ln_eps, dh, gw.g1, gw.be1, dz);
    /* z1 = x + W_o a + b_o */
    memcpy(dx, dz, sizeof(double) * nd);
    memset(da, 0, sizeof(double) * nd);
    linear_back(n, d, d, att + nd * l, w.Wo, dz, gw.Wo, gw.bo, da);
    /* a = attention(qkv) */
    memset(dq, 0, sizeof(double) * nd * 3);
    attention_back(c, n, Mk, qkv + nd * 3 * l, da, dq);
    /* qkv = W_qkv x + b_qkv */
    linear_back(n, d, 3 * d, xs + nd * l, w.Wqkv, dq, gw.Wqkv, gw.bqkv, dx);
  }
  /* x0 = W_in f + b_in + PE(depth): PE has no weights */
  linear_back(n, ORC_F, d, F, t.W_in, dx, gt.W_in, gt.b_in, NULL);
  free(depth); free(R); free(Mk); free(F); free(xs); free(qkv); free(att); free(z1); free(hh);
  free(up); free(uu); free(z2); free(g); free(a1); free(a2); free(r1); free(r2);
  free(dr2); free(dr1); free(dg); free(dx); free(dz); free(dh); free(du); free(da); free(dq);
  return ORC_OK;
}
