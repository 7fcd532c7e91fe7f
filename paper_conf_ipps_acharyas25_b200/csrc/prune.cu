// prune.cu -- graph pruning on the device (predtop_prune_graphs; SIV-B4,
// P:167-170): "There are several operations whose effects can
// be stored in the graph even after removing them ... such as reshape and
// convert_element_type ... We remove these redundant operators".
//
// Reading R21: an OPERATOR node whose op id is in the caller's
// set is removed; every other node is kept, renumbered in its original order
// with its record unchanged; kept u gets an edge to kept w iff the raw graph
// has a path u -> ... -> w (>= 1 edge) whose interior nodes are all removed.
// Output edges are unique and sorted by (src, dst) within each graph.
//
//   k_prune_meta   per-graph size checks and row offsets (one CTA)
//   k_prune_rows   one CTA per graph: validation, keep flags + new ids (block
//                  scan), successor CSR, Kahn levels (cycle check), then from
//                  the deepest level up the bitset over KEPT nodes
//                      P[v] = OR_{s in succ(v)} (kept(s) ? {id(s)} : P[s])
//                  (the closure recurrence of dag.cu with removed nodes made
//                  transparent); the edges of kept u are the bits of P[u]
//   k_prune_scan   output node / edge offsets (one CTA)
//   k_prune_emit   one CTA per graph: records of kept nodes, edges in (u, bit)
//                  order -- sorted and unique by construction
#include <climits>

#include "internal.h"

namespace predtop {

namespace {

template <class T>
__device__ T excl_scan(T v, T* total, T* sh /*[32]*/) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  T x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const T y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) sh[wid] = x;
  __syncthreads();
  if (wid == 0) {
    T w = lane < nw ? sh[lane] : T(0);
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const T y = __shfl_up_sync(0xffffffffu, w, o);
      if (lane >= o) w += y;
    }
    sh[lane] = w;
  }
  __syncthreads();
  const T base = wid > 0 ? sh[wid - 1] : T(0);
  *total = sh[nw - 1];
  __syncthreads();
  return base + x - v;
}

struct PruneDev {
  const int64_t* node_ptr;
  const int64_t* edge_ptr;
  const int32_t* src;
  const int32_t* dst;
  const predtop_node_feat* feats;
  uint16_t ops[PREDTOP_PRUNE_MAX_OPS];
  int n_ops;
  int max_nodes;
  int32_t* status;    // [G]
  int32_t* nk;        // [G] kept nodes
  int64_t* ne;        // [G] output edges
  int64_t* row_off;   // [G+1] prefix of N_g * ceil(N_g / 64)
  int32_t* first_bad; // [1]
  int64_t* totals;    // [2] nodes, edges
  int32_t* newid;     // [N_tot] -1 = removed
  int32_t* indeg;     // [N_tot]
  int32_t* soff;      // [N_tot + G]
  int32_t* succ;      // [E]
  int32_t* topo;      // [N_tot]
  int32_t* lptr;      // [N_tot + G]
  uint64_t* rows;     // [row_off[G]]
};

__global__ void __launch_bounds__(1024) k_prune_meta(PruneDev d, int G) {
  __shared__ int64_t sh[32];
  __shared__ int s_first;
  if (threadIdx.x == 0) s_first = INT_MAX;
  int64_t carry = 0;
  for (int base = 0; base < G; base += blockDim.x) {
    const int g = base + threadIdx.x;
    int64_t words = 0;
    if (g < G) {
      const int64_t n = d.node_ptr[g + 1] - d.node_ptr[g];
      const int64_t e = d.edge_ptr[g + 1] - d.edge_ptr[g];
      int st = PREDTOP_OK;
      if (n < 1 || n > d.max_nodes || n > PREDTOP_MAX_NODES) st = PREDTOP_ERR_TOO_LARGE;
      else if (e < 0) st = PREDTOP_ERR_INVALID_ARG;
      d.status[g] = st;
      d.nk[g] = 0;
      d.ne[g] = 0;
      if (st == PREDTOP_OK) words = n * ((n + 63) / 64);
    }
    int64_t tot;
    const int64_t ex = excl_scan<int64_t>(words, &tot, sh);
    if (g < G) d.row_off[g] = carry + ex;
    carry += tot;
  }
  __syncthreads();
  for (int g = threadIdx.x; g < G; g += blockDim.x)
    if (d.status[g] != PREDTOP_OK) atomicMin(&s_first, g);
  __syncthreads();
  if (threadIdx.x == 0) {
    d.row_off[G] = carry;
    *d.first_bad = s_first;
  }
}

__device__ __forceinline__ bool removed_op(const PruneDev& d, const predtop_node_feat& f) {
  if (f.kind != PREDTOP_KIND_OPERATOR) return false;
  bool hit = false;
  for (int i = 0; i < d.n_ops; ++i) hit |= f.op == d.ops[i];
  return hit;
}

__global__ void __launch_bounds__(256) k_prune_rows(PruneDev d) {
  const int g = blockIdx.x;
  if (d.status[g] != PREDTOP_OK) return;
  __shared__ int s_err, s_tail;
  __shared__ int32_t sh32[32];
  __shared__ unsigned long long s_edges;
  const int64_t n0 = d.node_ptr[g];
  const int N = (int)(d.node_ptr[g + 1] - n0);
  const int64_t e0 = d.edge_ptr[g];
  const int E = (int)(d.edge_ptr[g + 1] - e0);
  int32_t* newid = d.newid + n0;
  int32_t* indeg = d.indeg + n0;
  int32_t* soff = d.soff + n0 + g;
  int32_t* lptr = d.lptr + n0 + g;
  int32_t* succ = d.succ + e0;
  int32_t* topo = d.topo + n0;
  const int32_t* src = d.src + e0;
  const int32_t* dst = d.dst + e0;
  const int tid = threadIdx.x, nt = blockDim.x;
  if (tid == 0) { s_err = 0; s_tail = 0; s_edges = 0; soff[0] = 0; }
  for (int v = tid; v < N; v += nt) { indeg[v] = 0; soff[v + 1] = 0; }
  __syncthreads();
  for (int e = tid; e < E; e += nt) {
    const int s = src[e], t = dst[e];
    if (s < 0 || s >= N || t < 0 || t >= N) atomicOr(&s_err, 1);
    else if (s == t) atomicOr(&s_err, 2);
    else {
      atomicAdd(&indeg[t], 1);
      atomicAdd(&soff[s + 1], 1);
    }
  }
  __syncthreads();
  if (s_err) {
    if (tid == 0) {
      d.status[g] = (s_err & 1) ? PREDTOP_ERR_RANGE : PREDTOP_ERR_SELF_LOOP;
      atomicMin(d.first_bad, g);
    }
    return;
  }
  // keep flags and new ids (original order), kept count
  int32_t carry = 0;
  for (int base = 0; base < N; base += nt) {
    const int v = base + tid;
    const int k = (v < N && !removed_op(d, d.feats[n0 + v])) ? 1 : 0;
    int32_t tot;
    const int32_t ex = excl_scan<int32_t>(k, &tot, sh32);
    if (v < N) newid[v] = k ? carry + ex : -1;
    carry += tot;
  }
  const int NK = carry;
  // successor CSR
  carry = 0;
  for (int base = 0; base < N; base += nt) {
    const int v = base + tid;
    const int32_t c = v < N ? soff[v + 1] : 0;
    int32_t tot;
    const int32_t ex = excl_scan<int32_t>(c, &tot, sh32);
    if (v < N) soff[v + 1] = carry + ex + c;
    carry += tot;
  }
  __syncthreads();
  for (int v = tid; v < N; v += nt) lptr[v] = soff[v];
  __syncthreads();
  for (int e = tid; e < E; e += nt) succ[atomicAdd(&lptr[src[e]], 1)] = dst[e];
  __syncthreads();
  // Kahn levels (a graph whose order misses a node has a cycle)
  for (int v = tid; v < N; v += nt)
    if (indeg[v] == 0) topo[atomicAdd(&s_tail, 1)] = v;
  __syncthreads();
  int lb = 0, le = s_tail, level = 0;
  if (tid == 0) lptr[0] = 0;
  while (lb < le) {
    for (int i = lb + tid; i < le; i += nt) {
      const int v = topo[i];
      for (int k = soff[v]; k < soff[v + 1]; ++k)
        if (atomicSub(&indeg[succ[k]], 1) == 1) topo[atomicAdd(&s_tail, 1)] = succ[k];
    }
    __syncthreads();
    lb = le;
    le = s_tail;
    ++level;
    if (tid == 0) lptr[level] = lb;
    __syncthreads();
  }
  if (le != N) {
    if (tid == 0) {
      d.status[g] = PREDTOP_ERR_CYCLE;
      atomicMin(d.first_bad, g);
    }
    return;
  }
  if (tid == 0) d.nk[g] = NK;
  if (NK == 0) return;
  // rows over kept ids, deepest level first
  const int W = (NK + 63) / 64;
  uint64_t* P = d.rows + d.row_off[g];
  for (int l = level - 1; l >= 0; --l) {
    const int b = lptr[l], items = (lptr[l + 1] - b) * W;
    for (int it = tid; it < items; it += nt) {
      const int v = topo[b + it / W], j = it % W;
      uint64_t acc = 0;
      for (int k = soff[v]; k < soff[v + 1]; ++k) {
        const int s = succ[k];
        const int id = newid[s];
        if (id >= 0) acc |= ((id >> 6) == j) ? 1ull << (id & 63) : 0ull;
        else acc |= P[(int64_t)s * W + j];
      }
      P[(int64_t)v * W + j] = acc;
    }
    __syncthreads();
  }
  unsigned long long cnt = 0;
  for (int64_t it = tid; it < (int64_t)N * W; it += nt)
    if (newid[it / W] >= 0) cnt += __popcll(P[it]);
  atomicAdd(&s_edges, cnt);
  __syncthreads();
  if (tid == 0) d.ne[g] = (int64_t)s_edges;
}

__global__ void __launch_bounds__(1024) k_prune_scan(PruneDev d, int G, int64_t* out_node_ptr,
                                                     int64_t* out_edge_ptr) {
  __shared__ int64_t sh[32];
  int64_t cn = 0, ce = 0;
  for (int base = 0; base < G; base += blockDim.x) {
    const int g = base + threadIdx.x;
    const bool ok = g < G && d.status[g] == PREDTOP_OK;
    int64_t tot;
    int64_t ex = excl_scan<int64_t>(ok ? (int64_t)d.nk[g] : 0, &tot, sh);
    if (g < G) out_node_ptr[g] = cn + ex;
    cn += tot;
    ex = excl_scan<int64_t>(ok ? d.ne[g] : 0, &tot, sh);
    if (g < G) out_edge_ptr[g] = ce + ex;
    ce += tot;
  }
  if (threadIdx.x == 0) {
    out_node_ptr[G] = cn;
    out_edge_ptr[G] = ce;
    d.totals[0] = cn;
    d.totals[1] = ce;
  }
}

__global__ void __launch_bounds__(256) k_prune_emit(PruneDev d, const int64_t* out_node_ptr,
                                                    const int64_t* out_edge_ptr, int32_t* out_src,
                                                    int32_t* out_dst, predtop_node_feat* out_feats) {
  const int g = blockIdx.x;
  if (d.status[g] != PREDTOP_OK) return;
  __shared__ int64_t sh[32];
  const int64_t n0 = d.node_ptr[g];
  const int N = (int)(d.node_ptr[g + 1] - n0);
  const int NK = d.nk[g];
  if (NK == 0) return;
  const int W = (NK + 63) / 64;
  const int32_t* newid = d.newid + n0;
  const uint64_t* P = d.rows + d.row_off[g];
  const int64_t fo = out_node_ptr[g];
  int64_t eo = out_edge_ptr[g];
  for (int base = 0; base < N; base += blockDim.x) {
    const int v = base + threadIdx.x;
    const int id = v < N ? newid[v] : -1;
    int64_t cnt = 0;
    if (id >= 0) {
      out_feats[fo + id] = d.feats[n0 + v];
      for (int j = 0; j < W; ++j) cnt += __popcll(P[(int64_t)v * W + j]);
    }
    int64_t tot;
    int64_t pos = eo + excl_scan<int64_t>(cnt, &tot, sh);
    if (id >= 0)
      for (int j = 0; j < W; ++j) {
        uint64_t w = P[(int64_t)v * W + j];
        while (w) {
          const int b = __ffsll((long long)w) - 1;
          w &= w - 1;
          out_src[pos] = id;
          out_dst[pos] = j * 64 + b;
          ++pos;
        }
      }
    eo += tot;
  }
}

size_t carve_prune(const predtop_batch_desc* b, void* ws, PruneDev* o) {
  Carver c(ws);
  const int64_t G = b->num_graphs, N = b->total_nodes, E = std::max<int64_t>(b->total_edges, 1);
  const int64_t maxn = std::min<int64_t>(b->max_nodes, PREDTOP_MAX_NODES);
  PruneDev t{};
  t.status = c.take<int32_t>(G);
  t.nk = c.take<int32_t>(G);
  t.ne = c.take<int64_t>(G);
  t.row_off = c.take<int64_t>(G + 1);
  t.first_bad = c.take<int32_t>(1);
  t.totals = c.take<int64_t>(2);
  t.newid = c.take<int32_t>(N);
  t.indeg = c.take<int32_t>(N);
  t.soff = c.take<int32_t>(N + G);
  t.succ = c.take<int32_t>(E);
  t.topo = c.take<int32_t>(N);
  t.lptr = c.take<int32_t>(N + G);
  t.rows = c.take<uint64_t>((size_t)N * ceil_div(maxn, 64));
  if (o) *o = t;
  return align_up(c.used, 256);
}

}  // namespace

size_t prune_workspace_bytes(const predtop_batch_desc* b) { return carve_prune(b, nullptr, nullptr); }

predtop_status prune_launch(const predtop_batch_desc* b, const int64_t* node_ptr, const int64_t* edge_ptr,
                            const int32_t* src, const int32_t* dst, const predtop_node_feat* feats,
                            const uint16_t* ops, int n_ops, void* ws, int64_t* out_node_ptr,
                            int64_t* out_edge_ptr, int32_t* out_src, int32_t* out_dst,
                            int64_t edge_capacity, predtop_node_feat* out_feats, int64_t* totals_host,
                            int32_t* first_bad_host, cudaStream_t st) {
  PruneDev d{};
  carve_prune(b, ws, &d);
  d.node_ptr = node_ptr; d.edge_ptr = edge_ptr; d.src = src; d.dst = dst; d.feats = feats;
  for (int i = 0; i < n_ops; ++i) d.ops[i] = ops[i];
  d.n_ops = n_ops;
  d.max_nodes = b->max_nodes;
  const int G = b->num_graphs;
  {
    ProfScope _p(PK_PRUNE, st);
    k_prune_meta<<<1, 1024, 0, st>>>(d, G);
    PT_LAUNCH_CHECK();
    k_prune_rows<<<G, 256, 0, st>>>(d);
    PT_LAUNCH_CHECK();
    k_prune_scan<<<1, 1024, 0, st>>>(d, G, out_node_ptr, out_edge_ptr);
    PT_LAUNCH_CHECK();
  }
  int64_t tot[2];
  int32_t fb = INT_MAX;
  PT_CUDA_TRY(cudaMemcpyAsync(tot, d.totals, sizeof(tot), cudaMemcpyDeviceToHost, st));
  PT_CUDA_TRY(cudaMemcpyAsync(&fb, d.first_bad, sizeof(fb), cudaMemcpyDeviceToHost, st));
  PT_CUDA_TRY(cudaStreamSynchronize(st));
  if (totals_host) { totals_host[0] = tot[0]; totals_host[1] = tot[1]; }
  if (fb != INT_MAX) {
    int32_t s = PREDTOP_OK;
    PT_CUDA_TRY(cudaMemcpy(&s, d.status + fb, sizeof(s), cudaMemcpyDeviceToHost));
    if (first_bad_host) *first_bad_host = fb;
    set_error("prune: graph %d is invalid (status %d)", fb, s);
    return (predtop_status)s;
  }
  if (tot[1] > edge_capacity) {
    set_error("prune: %lld output edges > capacity %lld", (long long)tot[1], (long long)edge_capacity);
    return PREDTOP_ERR_WORKSPACE;
  }
  {
    ProfScope _p(PK_PRUNE, st);
    k_prune_emit<<<G, 256, 0, st>>>(d, out_node_ptr, out_edge_ptr, out_src, out_dst, out_feats);
    PT_LAUNCH_CHECK();
  }
  return PREDTOP_OK;
}

}  // namespace predtop
