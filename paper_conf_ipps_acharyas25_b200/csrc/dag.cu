// dag.cu -- stage-DAG preprocessing on the device (predtop_build_dag).
//
//  k_meta      per-graph sizes, size checks, prefix offsets (one CTA)
//  k_depth     K1: range / self-loop check, successor CSR, level-synchronous
//              Kahn (P:137 DAGPE depth = Kahn level = longest path from a
//              source; a graph whose Kahn order misses a node has a cycle)
//  k_closure   K2: packed-bitset transitive closure R[v] = OR_{w in succ(v)}
//              (R[w] | {w}), level-synchronous from the deepest level up
//              (P:135 DAGRA, P:145 k = infinity); one CTA per (graph, column
//              slice), the slice of all rows resident in shared memory
//  k_mask2     K3: M = R | R^T | I (stored layout) per 128-row block, rows
//              and column strip staged in shared memory, 32x32 bit transposes
//              by shuffles, popcounts per 128x128 tile
//  k_classify  tile classes (empty / partial / full) and |A| per graph
//  k_dag_small all of the above fused, one warp per graph (N <= 512)
//  k_bflags    16x64 attention block flags, mask words to the stored layout
// The attention work list (graph, 128-row q-tile) is written by k_meta.
#include <algorithm>
#include <climits>

#include "internal.h"

namespace predtop {

template <class T>
__device__ T block_excl_scan(T v, T* total, T* sh /*[32]*/) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  T x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) sh[wid] = x;
  __syncthreads();
  if (wid == 0) {
    T w = lane < nw ? sh[lane] : T(0);
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      T y = __shfl_up_sync(0xffffffffu, w, o);
      if (lane >= o) w += y;
    }
    sh[lane] = w;
  }
  __syncthreads();
  T base = wid > 0 ? sh[wid - 1] : T(0);
  *total = sh[nw - 1];
  __syncthreads();
  return base + x - v;
}

// Graphs with N <= sc.sn nodes take the fused one-warp-per-graph path
// (k_dag_small; its successor lists sit in shared memory when E <= sc.se, else
// in the global CSR scratch); the multi-kernel path below skips them.
struct SmallCfg {
  int sn, se, slot;  // node / edge capacity of a warp slot, slot bytes
};
__host__ __device__ inline bool is_small(int N, int /*E*/, const SmallCfg& sc) {
  return N <= sc.sn;
}

__global__ void __launch_bounds__(1024) k_meta(DagDev d, int G, int max_nodes) {
  __shared__ int64_t sh64[32];
  int64_t carry_rows = 0, carry_tiles = 0, carry_q = 0, carry_f = 0;
  for (int base = 0; base < G; base += blockDim.x) {
    const int g = base + threadIdx.x;
    int64_t rows = 0, tiles = 0, q = 0, fl = 0, n = 0;
    if (g < G) {
      n = d.node_ptr[g + 1] - d.node_ptr[g];
      const int64_t e = d.edge_ptr[g + 1] - d.edge_ptr[g];
      int st = PREDTOP_OK;
      if (n < 1 || n > max_nodes || n > PREDTOP_MAX_NODES) st = PREDTOP_ERR_TOO_LARGE;
      else if (e < 0) st = PREDTOP_ERR_INVALID_ARG;
      d.status[g] = st;
      d.num_levels[g] = 0;
      d.pairs[g] = 0;
      if (st == PREDTOP_OK) {
        const int64_t T = (n + 127) / 128;
        rows = n * 2 * T;
        tiles = T * T;
        q = T;
        fl = ((n + 15) / 16) * ((n + 63) / 64);
      }
    }
    int64_t tot;
    int64_t ex = block_excl_scan<int64_t>(rows, &tot, sh64);
    if (g < G) d.row_off[g] = carry_rows + ex;
    carry_rows += tot;
    ex = block_excl_scan<int64_t>(tiles, &tot, sh64);
    if (g < G) d.tile_off[g] = carry_tiles + ex;
    carry_tiles += tot;
    ex = block_excl_scan<int64_t>(q, &tot, sh64);
    if (g < G) {
      // attention work items (graph, 128-row q-tile), written for every graph
      // with rows here, so a graph that a later kernel marks RANGE / SELF_LOOP /
      // CYCLE still leaves valid items (attention skips it by its status)
      d.qtile_off[g] = (int32_t)(carry_q + ex);
      for (int qt = 0; qt < q; ++qt) d.work[carry_q + ex + qt] = make_int2(g, qt);
    }
    carry_q += tot;
    ex = block_excl_scan<int64_t>(fl, &tot, sh64);
    if (g < G) d.bflag_off[g] = carry_f + ex;
    carry_f += tot;
  }
  // lowest graph with a size error (device-detected errors lower it later)
  __shared__ int s_first;
  if (threadIdx.x == 0) s_first = INT_MAX;
  __syncthreads();
  for (int g = threadIdx.x; g < G; g += blockDim.x)
    if (d.status[g] != PREDTOP_OK) atomicMin(&s_first, g);
  __syncthreads();
  if (threadIdx.x == 0) {
    d.row_off[G] = carry_rows;
    d.tile_off[G] = carry_tiles;
    d.qtile_off[G] = (int32_t)carry_q;
    d.bflag_off[G] = carry_f;
    *d.first_bad = s_first;
  }
}

// K1: validation + successor CSR + Kahn levels / depth.  One CTA per graph.
// With `smem_nodes` >= N the in-degree counters and the Kahn queue live in
// shared memory (the per-level atomicSub and the frontier reads are then
// shared-memory round trips, not L2 ones: a deep graph runs ~11k levels)
// and the queue is copied to global (topo) at the end.
__global__ void __launch_bounds__(256) k_depth(DagDev d, SmallCfg sc, int smem_nodes, int ecap) {
  extern __shared__ __align__(16) int32_t sm_depth[];
  const int g = blockIdx.x;
  if (d.status[g] != PREDTOP_OK) return;
  if (is_small((int)(d.node_ptr[g + 1] - d.node_ptr[g]), (int)(d.edge_ptr[g + 1] - d.edge_ptr[g]), sc)) return;
  __shared__ int s_err, s_tail;
  __shared__ int32_t sh32[32];
  const int64_t n0 = d.node_ptr[g];
  const int N = (int)(d.node_ptr[g + 1] - n0);
  const int64_t e0 = d.edge_ptr[g];
  const int E = (int)(d.edge_ptr[g + 1] - e0);
  const bool in_smem = N <= smem_nodes;
  int32_t* indeg = in_smem ? sm_depth : d.indeg + n0;
  int32_t* soff = d.succ_off + n0 + g;   // N+1
  int32_t* lptr = d.level_ptr + n0 + g;  // N+1 (first used as fill cursor)
  int32_t* succ = d.succ + e0;
  int32_t* const topo_g = d.topo + n0;
  int32_t* topo = in_smem ? sm_depth + smem_nodes : topo_g;
  int32_t* depth = d.depth + n0;
  const int32_t* src = d.src + e0;
  const int32_t* dst = d.dst + e0;
  const int tid = threadIdx.x, nt = blockDim.x;

  if (tid == 0) { s_err = 0; s_tail = 0; soff[0] = 0; }
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
    for (int v = tid; v < N; v += nt) depth[v] = -1;
    return;
  }
  // inclusive scan of out-degrees -> soff[1..N]
  int32_t carry = 0;
  for (int base = 0; base < N; base += nt) {
    const int v = base + tid;
    const int32_t c = v < N ? soff[v + 1] : 0;
    int32_t tot;
    const int32_t ex = block_excl_scan<int32_t>(c, &tot, sh32);
    if (v < N) soff[v + 1] = carry + ex + c;
    carry += tot;
  }
  __syncthreads();
  for (int v = tid; v < N; v += nt) lptr[v] = soff[v];
  __syncthreads();
  for (int e = tid; e < E; e += nt) {
    const int pos = atomicAdd(&lptr[src[e]], 1);
    succ[pos] = dst[e];
  }
  __syncthreads();
  // Kahn, level synchronous: a node enters level l+1 when its last
  // predecessor (at level l) is retired, so its level is 1 + max pred level.
  int lb = 0, le = 0, level = 0;
  if (in_smem && N < 65536 && E <= ecap) {
    // Warp mode: the CSR as 16-bit arrays in shared memory and ONE warp
    // walking the levels with warp barriers (ballot + prefix-popcount queue
    // appends): deep graphs (16k nodes: ~11k levels of one or two nodes)
    // are a chain of dependent level steps, each a few shared-memory round
    // trips instead of global loads and two CTA barriers.
    uint16_t* topo16 = reinterpret_cast<uint16_t*>(sm_depth + smem_nodes);
    uint16_t* soff16 = topo16 + smem_nodes;
    uint16_t* succ16 = soff16 + smem_nodes + 1;
    for (int v = tid; v <= N; v += nt) soff16[v] = (uint16_t)soff[v];
    for (int e = tid; e < E; e += nt) succ16[e] = (uint16_t)succ[e];
    __syncthreads();
    if (tid < 32) {
      const int lane = tid;
      const uint32_t lt = (1u << lane) - 1u;
      int tail = 0;
      for (int base = 0; base < N; base += 32) {
        const int v = base + lane;
        const bool z = v < N && indeg[v] == 0;
        const uint32_t bal = __ballot_sync(0xffffffffu, z);
        if (z) {
          topo16[tail + __popc(bal & lt)] = (uint16_t)v;
          depth[v] = 0;
        }
        tail += __popc(bal);
      }
      if (lane == 0) lptr[0] = 0;
      __syncwarp();
      int wb = 0, we = tail, wl = 0;
      while (wb < we) {
        for (int i0 = wb; i0 < we; i0 += 32) {
          int k = 0, kend = 0;
          if (i0 + lane < we) {
            const int v = topo16[i0 + lane];
            k = soff16[v];
            kend = soff16[v + 1];
          }
          while (__any_sync(0xffffffffu, k < kend)) {
            int w = 0;
            bool ready = false;
            if (k < kend) {
              w = succ16[k++];
              ready = atomicSub(&indeg[w], 1) == 1;
            }
            const uint32_t bal = __ballot_sync(0xffffffffu, ready);
            if (ready) {
              topo16[tail + __popc(bal & lt)] = (uint16_t)w;
              depth[w] = wl + 1;
            }
            tail += __popc(bal);
          }
        }
        __syncwarp();
        wb = we;
        we = tail;
        ++wl;
        if (lane == 0) lptr[wl] = wb;
      }
      if (lane == 0) { s_tail = we; sh32[0] = wl; }
    }
    __syncthreads();
    le = s_tail;
    level = sh32[0];
    for (int i = tid; i < le; i += nt) topo_g[i] = topo16[i];
    __syncthreads();
    topo = topo_g;
  } else {
  for (int v = tid; v < N; v += nt)
    if (indeg[v] == 0) {
      const int p = atomicAdd(&s_tail, 1);
      topo[p] = v;
      depth[v] = 0;
    }
  __syncthreads();
  le = s_tail;
  if (tid == 0) lptr[0] = 0;
  while (lb < le) {
    for (int i = lb + tid; i < le; i += nt) {
      const int v = topo[i];
      for (int k = soff[v]; k < soff[v + 1]; ++k) {
        const int w = succ[k];
        if (atomicSub(&indeg[w], 1) == 1) {
          const int p = atomicAdd(&s_tail, 1);
          topo[p] = w;
          depth[w] = level + 1;
        }
      }
    }
    __syncthreads();
    lb = le;  // level `level` spans topo[lptr[level] .. lptr[level+1])
    le = s_tail;
    ++level;
    if (tid == 0) lptr[level] = lb;
    __syncthreads();
  }
  if (in_smem)
    for (int i = tid; i < le; i += nt) topo_g[i] = topo[i];
  }  // block-synchronous mode
  if (tid == 0) d.num_levels[g] = level;
  if (le == N) {  // closure records in topo order: node, degree, first four successors inline
    int4* rec = d.rec + n0;
    for (int i = tid; i < N; i += nt) {
      const int v = topo[i];
      const int b = soff[v], deg = soff[v + 1] - b;
      int s4[4] = {0, 0, 0, 0};
      for (int k = 0; k < 4 && k < deg; ++k) s4[k] = succ[b + k];
      rec[i] = make_int4(v | (min(deg, 0xFFFF) << 16), s4[0] | (s4[1] << 16), s4[2] | (s4[3] << 16), b);
    }
  }
  if (le != N) {
    if (tid == 0) {
      d.status[g] = PREDTOP_ERR_CYCLE;
      atomicMin(d.first_bad, g);
    }
    for (int v = tid; v < N; v += nt) depth[v] = -1;
  }
}

#ifndef PREDTOP_CLOS_REC_SMEM
#define PREDTOP_CLOS_REC_SMEM 1  // k_closure level loop over shared-memory records (0: over the CSR)
#endif
#ifndef PREDTOP_REC_AHEAD
#define PREDTOP_REC_AHEAD 4
#endif
constexpr int kRecAhead = PREDTOP_REC_AHEAD;  // closure record prefetch distance (levels)

// K2: closure.  grid = (G, slices); dynamic smem `smem_bytes`.
__global__ void __launch_bounds__(256) k_closure(DagDev d, int smem_bytes, SmallCfg sc) {
  extern __shared__ __align__(16) unsigned char sm[];
  const int g = blockIdx.x, slice = blockIdx.y;
  const int64_t n0 = d.node_ptr[g];
  const int N = (int)(d.node_ptr[g + 1] - n0);
  if (is_small(N, (int)(d.edge_ptr[g + 1] - d.edge_ptr[g]), sc)) return;
  const int st = d.status[g];
  if (st == PREDTOP_ERR_TOO_LARGE || st == PREDTOP_ERR_INVALID_ARG) return;  // no rows
  const int W = 2 * ((N + 127) / 128);
  uint64_t* Rg = d.R + d.row_off[g];
  const int tid = threadIdx.x, nt = blockDim.x;
  // Column slicing: CW words of every row resident in shared memory.
  const int L = d.num_levels[g];
  const int E = (int)(d.edge_ptr[g + 1] - d.edge_ptr[g]);
  // finite-k rounds read the CSR; the k = infinity level loop reads the
  // per-node records (node, degree, first four successors, in topo order;
  // built by k_depth) and the level bounds
  const bool kfin = d.hops > 0 && d.hops < L - 1;
  const bool recs = !kfin && PREDTOP_CLOS_REC_SMEM;
  const size_t csr_bytes = recs ? align_up((size_t)16 * N + 4 * ((size_t)L + 1), 16)
                                : align_up((size_t)4 * ((size_t)N + (N + 1) + E + (L + 1)), 16);
  int CW = (int)min((int64_t)W, (int64_t)smem_bytes / (8 * (int64_t)N));
  bool csr_in_smem = false;
  if ((int64_t)smem_bytes > (int64_t)csr_bytes) {
    const int cw2 = (int)min((int64_t)W, ((int64_t)smem_bytes - (int64_t)csr_bytes) / (8 * (int64_t)N));
    if (cw2 >= 1 && (W + cw2 - 1) / cw2 <= (int)gridDim.y) { CW = cw2; csr_in_smem = true; }
  }
  const bool global_mode = CW < 1;
  if (global_mode) CW = max(1, (W + (int)gridDim.y - 1) / (int)gridDim.y);
  const int word0 = slice * CW;
  if (word0 >= W) return;
  const int nw = min(CW, W - word0);
  if (st != PREDTOP_OK) {  // device-detected error: rows are defined as zero
    for (int64_t it = tid; it < (int64_t)N * nw; it += nt)
      Rg[(it / nw) * W + word0 + it % nw] = 0;
    return;
  }
  const int32_t* topo = d.topo + n0;
  const int32_t* soff = d.succ_off + n0 + g;
  const int32_t* succ = d.succ + d.edge_ptr[g];
  const int32_t* lptr = d.level_ptr + n0 + g;
  const int K = d.hops;
  if (!csr_in_smem && !global_mode && !(K > 0 && K < L - 1)) {
    // Deep graphs whose CSR does not fit next to the slice (e.g. 16k nodes,
    // ~11k levels; for MoE-size graphs the CSR-in-SMEM loop below measured
    // faster: 1.27 vs 1.64 ms/step).  Level loop over per-node records (node, degree, first four successors;
    // built by k_depth in topo order) prefetched four levels ahead into
    // registers, and the level bounds from a shared-memory copy: the loop is
    // latency-bound (fwd+bwd stage graphs have ~N/3 levels of a few nodes),
    // so no dependent L2 round trip per level.  Bit columns are independent
    // (column j of R[v] reads column j of the successors' rows only), so each
    // warp owns the words j = warp, warp + nwarps, ... of the slice and walks
    // the levels on its own with warp barriers: no CTA barrier per level.
    uint64_t* Rsm = reinterpret_cast<uint64_t*>(sm);
    const int rs2 = CW;
    const size_t slice_bytes = align_up((size_t)N * CW * 8, 16);
    const bool lptr_smem = slice_bytes + (size_t)4 * (L + 1) <= (size_t)smem_bytes;
    int32_t* s_lp = reinterpret_cast<int32_t*>(sm + slice_bytes);
    if (lptr_smem)
      for (int i = tid; i <= L; i += nt) s_lp[i] = lptr[i];
    const int32_t* lp = lptr_smem ? s_lp : lptr;
    const int4* rec = d.rec + n0;
    for (int64_t it = tid; it < (int64_t)N * nw; it += nt) Rsm[(it / nw) * rs2 + it % nw] = 0;
    __syncthreads();
    const int warp = tid >> 5, lane = tid & 31, nwarps = nt >> 5;
    const int my_nw = warp < nw ? (nw - warp + nwarps - 1) / nwarps : 0;
    // i / my_nw as a multiply-high by ceil(2^32 / my_nw) (exact for i < 2^32 / my_nw)
    const uint32_t inv_nw = my_nw > 1 ? (uint32_t)((0xFFFFFFFFull + (uint64_t)my_nw) / (uint64_t)my_nw) : 0u;
    if (my_nw > 0) {
      auto first_rec = [&](int l) -> int4 {  // this lane's first item of level l
        if (l < 0) return make_int4(0, 0, 0, 0);
        const int b = lp[l], e = lp[l + 1];
        return lane < (e - b) * my_nw ? __ldg(rec + b + (my_nw == 1 ? lane : (int)__umulhi((uint32_t)lane, inv_nw)))
                                      : make_int4(0, 0, 0, 0);
      };
      // level `level` with its prefetched first record r0; then r0 <- the
      // record of level - 4 (four fixed registers, unrolled by four: a load is
      // only waited for when its level comes up)
      auto do_level = [&](int level, int4& r0) {
        const int lb = lp[level], items = (lp[level + 1] - lb) * my_nw;
        for (int i = lane; i < items; i += 32) {
          const int node_i = my_nw == 1 ? i : (int)__umulhi((uint32_t)i, inv_nw);
          const int4 r = i == lane ? r0 : __ldg(rec + lb + node_i);
          const uint32_t v = (uint32_t)r.x & 0xFFFFu, deg = (uint32_t)r.x >> 16;
          const int j = warp + (my_nw == 1 ? 0 : (i - node_i * my_nw)) * nwarps;
          const uint32_t wj = (uint32_t)(word0 + j);
          const uint32_t s4[4] = {(uint32_t)r.y & 0xFFFFu, (uint32_t)r.y >> 16, (uint32_t)r.z & 0xFFFFu,
                                  (uint32_t)r.z >> 16};
          uint64_t acc = 0;
#pragma unroll
          for (int k = 0; k < 4; ++k)
            if ((uint32_t)k < deg) {
              const uint32_t w = s4[k];
              acc |= Rsm[(size_t)w * rs2 + j] | ((w >> 6) == wj ? 1ull << (w & 63) : 0ull);
            }
          if (deg > 4) {
            const uint32_t dg = deg == 0xFFFFu ? (uint32_t)(soff[v + 1] - r.w) : deg;
            for (uint32_t k = 4; k < dg; ++k) {
              const uint32_t w = (uint32_t)succ[r.w + k];
              acc |= Rsm[(size_t)w * rs2 + j] | ((w >> 6) == wj ? 1ull << (w & 63) : 0ull);
            }
          }
          Rsm[(size_t)v * rs2 + j] = acc;
        }
        r0 = first_rec(level - kRecAhead);
        __syncwarp();
      };
      // records kRecAhead levels ahead (fixed registers, loop unrolled by
      // kRecAhead): the ~100-cycle level step would otherwise wait for an L2
      // round trip (600+ cycles) every few levels
      int4 rr[kRecAhead];
#pragma unroll
      for (int i = 0; i < kRecAhead; ++i) rr[i] = first_rec(L - 1 - i);
      for (int level = L - 1; level >= 0; level -= kRecAhead) {
#pragma unroll
        for (int i = 0; i < kRecAhead; ++i)
          if (level - i >= 0) do_level(level - i, rr[i]);
      }
    }
    __syncthreads();
    for (int64_t it = tid; it < (int64_t)N * nw; it += nt)
      Rg[(it / nw) * W + word0 + it % nw] = Rsm[(it / nw) * rs2 + it % nw];
    return;
  }
  uint64_t* Rs;
  int64_t rs;  // row stride of Rs in words
  const int32_t* soff_g = soff;
  const int32_t* succ_g = succ;
  const int4* s_rec = reinterpret_cast<const int4*>(sm);
  if (csr_in_smem && recs) {
    int4* rs_ = reinterpret_cast<int4*>(sm);
    int32_t* s_lptr = reinterpret_cast<int32_t*>(rs_ + N);
    const int4* rec = d.rec + n0;
    for (int i = tid; i < N; i += nt) rs_[i] = rec[i];
    for (int i = tid; i <= L; i += nt) s_lptr[i] = lptr[i];
    lptr = s_lptr;
  } else if (csr_in_smem) {
    int32_t* s_topo = (int32_t*)sm;
    int32_t* s_soff = s_topo + N;
    int32_t* s_succ = s_soff + (N + 1);
    int32_t* s_lptr = s_succ + E;
    for (int i = tid; i < N; i += nt) s_topo[i] = topo[i];
    for (int i = tid; i <= N; i += nt) s_soff[i] = soff[i];
    for (int i = tid; i < E; i += nt) s_succ[i] = succ[i];
    for (int i = tid; i <= L; i += nt) s_lptr[i] = lptr[i];
    topo = s_topo; soff = s_soff; succ = s_succ; lptr = s_lptr;
  }
  if (global_mode) {
    Rs = Rg + word0;
    rs = W;
  } else {
    Rs = (uint64_t*)(sm + (csr_in_smem ? csr_bytes : 0));
    rs = CW;
  }
  if (K > 0 && K < L - 1) {
    __syncthreads();  // the staged CSR above
    // finite-k DAGRA: K synchronous rounds over all rows,
    // R_j[v] = OR_{w in succ(v)} ({w} | R_{j-1}[w]), R_0 = 0, ping-ponging
    // between Rs and a second buffer of the same column slice (the global R
    // rows when Rs is shared memory, else the M rows, which k_mask2 rewrites
    // later); round j writes Rs iff K - j is even, so R_K ends in Rs.
    uint64_t* Xs = global_mode ? d.M + d.row_off[g] + word0 : Rg + word0;
    const int64_t xs = W;
    for (int j = 1; j <= K; ++j) {
      const bool to_rs = ((K - j) & 1) == 0;
      for (int64_t it = tid; it < (int64_t)N * nw; it += nt) {
        const int v = (int)(it / nw), c = (int)(it % nw);
        const int word = word0 + c;
        uint64_t acc = 0;
        for (int k = soff[v]; k < soff[v + 1]; ++k) {
          const int w = succ[k];
          if (j > 1) acc |= to_rs ? __ldcg(Xs + (int64_t)w * xs + c)
                                  : (global_mode ? __ldcg(Rs + (int64_t)w * rs + c) : Rs[(int64_t)w * rs + c]);
          if ((w >> 6) == word) acc |= 1ull << (w & 63);
        }
        if (to_rs) Rs[(int64_t)v * rs + c] = acc;
        else Xs[(int64_t)v * xs + c] = acc;
      }
      __threadfence();
      __syncthreads();
    }
  } else {
  for (int64_t it = tid; it < (int64_t)N * nw; it += nt) Rs[(it / nw) * rs + it % nw] = 0;
  __syncthreads();
  // Bit columns are independent (R[v] column j only reads column j of the
  // successors' rows), so each warp owns the words j = warp, warp + nwarps,
  // ... of the slice and walks the levels on its own with warp barriers: no
  // CTA barrier per level (the levels of fwd+bwd stage graphs hold a few
  // nodes, so the loop is latency-bound; 8 independent warps instead of one
  // CTA-synchronous sweep).
  const int warp = tid >> 5, lane = tid & 31, nwarps = nt >> 5;
  const int my_nw = warp < nw ? (nw - warp + nwarps - 1) / nwarps : 0;
  // it / my_nw as a multiply-high by ceil(2^32 / my_nw) (exact for it <
  // 2^32 / my_nw, far above N * my_nw): a runtime integer division is a ~20-instruction dependent chain
  // inside the latency-bound level step
  const uint32_t inv_nw = my_nw > 1 ? (uint32_t)((0xFFFFFFFFull + (uint64_t)my_nw) / (uint64_t)my_nw) : 0u;
  if (my_nw > 0 && csr_in_smem && recs) {
    // records in shared memory: one record load, then the successors' words
    for (int level = L - 1; level >= 0; --level) {
      const int lb = lptr[level], items = (lptr[level + 1] - lb) * my_nw;
      for (int it = lane; it < items; it += 32) {
        const int node_i = my_nw == 1 ? it : (int)__umulhi((uint32_t)it, inv_nw);
        const int j = warp + (my_nw == 1 ? 0 : it - node_i * my_nw) * nwarps;
        const uint32_t wj = (uint32_t)(word0 + j);
        const int4 r = s_rec[lb + node_i];
        const uint32_t v = (uint32_t)r.x & 0xFFFFu, deg = (uint32_t)r.x >> 16;
        const uint32_t s4[4] = {(uint32_t)r.y & 0xFFFFu, (uint32_t)r.y >> 16, (uint32_t)r.z & 0xFFFFu,
                                (uint32_t)r.z >> 16};
        uint64_t acc = 0;
#pragma unroll
        for (int k = 0; k < 4; ++k)
          if ((uint32_t)k < deg) {
            const uint32_t w = s4[k];
            acc |= Rs[(int64_t)w * rs + j] | ((w >> 6) == wj ? 1ull << (w & 63) : 0ull);
          }
        if (deg > 4) {
          const uint32_t dg = deg == 0xFFFFu ? (uint32_t)(soff_g[v + 1] - r.w) : deg;
          for (uint32_t k = 4; k < dg; ++k) {
            const uint32_t w = (uint32_t)succ_g[r.w + k];
            acc |= Rs[(int64_t)w * rs + j] | ((w >> 6) == wj ? 1ull << (w & 63) : 0ull);
          }
        }
        Rs[(int64_t)v * rs + j] = acc;
      }
      __syncwarp();
    }
  } else if (my_nw > 0) {
    for (int level = L - 1; level >= 0; --level) {
      const int lb = lptr[level], le = lptr[level + 1];
      const int items = (le - lb) * my_nw;
      for (int it = lane; it < items; it += 32) {
        const int v = topo[lb + it / my_nw];
        const int j = warp + (it % my_nw) * nwarps;
        const int word = word0 + j;
        uint64_t acc = 0;
        for (int k = soff[v]; k < soff[v + 1]; ++k) {
          const int w = succ[k];
          acc |= Rs[(int64_t)w * rs + j];
          if ((w >> 6) == word) acc |= 1ull << (w & 63);
        }
        Rs[(int64_t)v * rs + j] = acc;
      }
      __syncwarp();
    }
  }
  __syncthreads();
  }
  if (!global_mode)
    for (int64_t it = tid; it < (int64_t)N * nw; it += nt)
      Rg[(it / nw) * W + word0 + it % nw] = Rs[(it / nw) * rs + it % nw];
}

// 32x32 bit-matrix transpose across a warp: lane i holds row i (bit j =
// column j) on entry and column i (bit j = row j) on exit.  Five butterfly
// stages of shuffles with swap masks (instead of 32 ballots).
__device__ __forceinline__ uint32_t transpose32(uint32_t x, int lane) {
#pragma unroll
  for (int k = 0; k < 5; ++k) {
    const int sh = 16 >> k;
    const uint32_t m = k == 0 ? 0x0000FFFFu : k == 1 ? 0x00FF00FFu : k == 2 ? 0x0F0F0F0Fu
                     : k == 3 ? 0x33333333u : 0x55555555u;
    const uint32_t y = __shfl_xor_sync(0xffffffffu, x, sh);
    x = (lane & sh) ? ((x & ~m) | ((y >> sh) & m)) : ((x & m) | ((y << sh) & ~m));
  }
  return x;
}

// K2 for deep graphs (the batch's largest graph has more than kDeepNodes
// nodes, k = infinity): 16-bit column chains.  Column j of R[v] only reads
// column j of the successors' rows, so every 16-bit column of R is an
// independent chain over the levels (deepest first).  A chain keeps its
// column for all N rows in shared memory (2 N bytes) and is walked by one
// warp: `cpb` chains per CTA, one CTA per SM, so the 4 W chains of a 16k-node
// graph (1024) run in ONE wave of 147 CTAs (64-bit column slices of 8 N bytes
// fit one per SM: two waves).  The walk is a chain of dependent level steps
// (~N/1.5 levels), so the number of chains in flight is what matters.  Level
// records (node, degree, first four successors; built by k_depth in topo
// order) and level bounds are prefetched kRecAhead levels ahead.
#ifndef PREDTOP_DEEP_NODES
#define PREDTOP_DEEP_NODES 6144
#endif
constexpr int kDeepNodes = PREDTOP_DEEP_NODES;
#ifndef PREDTOP_REC_AHEAD16
#define PREDTOP_REC_AHEAD16 4
#endif
constexpr int kRecAhead16 = PREDTOP_REC_AHEAD16;  // record prefetch distance (levels): ~L2 latency / level step
__global__ void __launch_bounds__(256) k_closure16(DagDev d, SmallCfg sc, int cpb) {
  extern __shared__ __align__(16) unsigned char sm_c16[];
  uint16_t* Rs = reinterpret_cast<uint16_t*>(sm_c16);  // [cpb][N]
  const int g = blockIdx.x;
  const int64_t n0 = d.node_ptr[g];
  const int N = (int)(d.node_ptr[g + 1] - n0);
  if (is_small(N, (int)(d.edge_ptr[g + 1] - d.edge_ptr[g]), sc)) return;
  const int st = d.status[g];
  if (st == PREDTOP_ERR_TOO_LARGE || st == PREDTOP_ERR_INVALID_ARG) return;  // no rows
  const int W = 2 * ((N + 127) / 128), nch = 4 * W;
  const int c0 = blockIdx.y * cpb;
  if (c0 >= nch) return;
  const int act = min(cpb, nch - c0);
  uint16_t* R16 = reinterpret_cast<uint16_t*>(d.R + d.row_off[g]);
  const int tid = threadIdx.x, nt = blockDim.x, warp = tid >> 5, lane = tid & 31;
  if (st != PREDTOP_OK) {  // device-detected error: rows are defined as zero
    for (int64_t it = tid; it < (int64_t)N * act; it += nt)
      R16[(it / act) * nch + c0 + it % act] = 0;
    return;
  }
  for (int64_t it = tid; it < (int64_t)N * act; it += nt) Rs[it] = 0;
  __syncthreads();
  if (warp < act) {
    const int L = d.num_levels[g];
    const int32_t* lp = d.level_ptr + n0 + g;
    const int32_t* soff = d.succ_off + n0 + g;
    const int32_t* succ = d.succ + d.edge_ptr[g];
    const int4* rec = d.rec + n0;
    uint16_t* col = Rs + (size_t)warp * N;
    const uint32_t cj = (uint32_t)(c0 + warp);  // this chain's 16 columns: [16 cj, +16)
    // Level bounds in registers, 32 levels per batch: lane j of batch q
    // holds lp[l] and lp[l + 1] of level l = L - 1 - 32 q - j; the batch
    // after the current one is loaded 32 levels ahead, and a level's bounds
    // are two shuffles (a global load here would put an L2 round trip on
    // every level step: the record fetch below depends on them)
    int q = 0, bc = 0, ec = 0, bn = 0, en = 0;
    auto load_batch = [&](int qq, int& bb, int& ee) {
      const int l = L - 1 - 32 * qq - lane;
      bb = l >= 0 ? __ldg(lp + l) : 0;
      ee = l >= 0 ? __ldg(lp + l + 1) : 0;
    };
    load_batch(0, bc, ec);
    load_batch(1, bn, en);
    auto bounds = [&](int l) -> int2 {  // l in batch q or q + 1 (warp-uniform)
      const int j = L - 1 - l - 32 * q;
      if (j < 32) return make_int2(__shfl_sync(0xffffffffu, bc, j), __shfl_sync(0xffffffffu, ec, j));
      return make_int2(__shfl_sync(0xffffffffu, bn, j - 32), __shfl_sync(0xffffffffu, en, j - 32));
    };
    // this lane's record of level l, kRecAhead16 levels ahead
    auto fetch = [&](int l, int4& r, int2& be) {
      if (l < 0) {
        r = make_int4(0, 0, 0, 0);
        be = make_int2(0, 0);
        return;
      }
      be = bounds(l);
      r = lane < be.y - be.x ? __ldg(rec + be.x + lane) : make_int4(0, 0, 0, 0);
    };
    auto do_level = [&](int level, int4& r0, int2& be0) {
      const int lb = be0.x, items = be0.y - be0.x;
      for (int i = lane; i < items; i += 32) {
        const int4 r = i == lane ? r0 : __ldg(rec + lb + i);
        const uint32_t v = (uint32_t)r.x & 0xFFFFu, deg = (uint32_t)r.x >> 16;
        const uint32_t s4[4] = {(uint32_t)r.y & 0xFFFFu, (uint32_t)r.y >> 16, (uint32_t)r.z & 0xFFFFu,
                                (uint32_t)r.z >> 16};
        uint32_t acc = 0;
#pragma unroll
        for (int k = 0; k < 4; ++k)
          if ((uint32_t)k < deg) {
            const uint32_t w = s4[k];
            acc |= col[w] | ((w >> 4) == cj ? 1u << (w & 15) : 0u);
          }
        if (deg > 4) {
          const uint32_t dg = deg == 0xFFFFu ? (uint32_t)(soff[v + 1] - r.w) : deg;
          for (uint32_t k = 4; k < dg; ++k) {
            const uint32_t w = (uint32_t)succ[r.w + k];
            acc |= col[w] | ((w >> 4) == cj ? 1u << (w & 15) : 0u);
          }
        }
        col[v] = (uint16_t)acc;
      }
      if (L - 1 - (level - kRecAhead16) - 32 * q >= 64) {  // the prefetch target left batch q + 1
        bc = bn;
        ec = en;
        ++q;
        load_batch(q + 1, bn, en);
      }
      fetch(level - kRecAhead16, r0, be0);
      __syncwarp();
    };
    int4 rr[kRecAhead16];
    int2 bb[kRecAhead16];
#pragma unroll
    for (int i = 0; i < kRecAhead16; ++i) fetch(L - 1 - i, rr[i], bb[i]);
    for (int level = L - 1; level >= 0; level -= kRecAhead16) {
#pragma unroll
      for (int i = 0; i < kRecAhead16; ++i)
        if (level - i >= 0) do_level(level - i, rr[i], bb[i]);
    }
  }
  __syncthreads();
  // rows out: consecutive threads write consecutive 16-bit columns of a row
  for (int64_t it = tid; it < (int64_t)N * act; it += nt) {
    const int64_t v = it / act;
    const int k = (int)(it - v * act);
    R16[v * nch + c0 + k] = Rs[(size_t)k * N + v];
  }
}

// K3 (large graphs): M = R | R^T | I in the stored layout and per-tile
// popcounts.  grid = (G, row blocks of 128), 8 warps.  A CTA owns M rows
// [128a, +128): the R rows of the block (column chunks of kMC words) and the
// R column strip of the block (words 2a, 2a+1 of every row v, i.e. the bits of
// columns u in the block) are staged in shared memory with coalesced loads,
// the strip is transposed in 32x32-bit tiles by shuffles and ORed into the
// rows, and the rows leave coalesced (mask_perm per 64-bit word).  The tile
// counts of row block a are this CTA's alone (no atomics in global memory).
// (The warp-per-32x32-block k_mask it replaces read and wrote one 32-bit word
// per 192-byte row per lane: 0.54 ms/step on MoE.)
constexpr int kMC = 32;           // 64-bit words per column chunk
constexpr int kMA = 2 * kMC + 1;  // padded row stride (32-bit words) of the row tile
constexpr int kMB = 5;            // padded row stride (32-bit words) of the strip
constexpr size_t kMaskSmem = (size_t)4 * (128 * kMA + 64 * kMC * kMB + 128);
__global__ void __launch_bounds__(256) k_mask2(DagDev d, SmallCfg sc, int rb) {
  extern __shared__ __align__(16) unsigned char sm_mask[];
  uint32_t* sA = reinterpret_cast<uint32_t*>(sm_mask);       // [128][kMA]
  uint32_t* sB = sA + 128 * kMA;                               // [64 kMC][kMB]
  int* s_cnt = reinterpret_cast<int*>(sB + 64 * kMC * kMB);  // [T <= 128]
  // row blocks of one graph are consecutive CTAs, so the graph's R column
  // strips, which every row block reads, are re-read from L2, not DRAM
  const int a = (int)(blockIdx.x % (unsigned)rb), g = (int)(blockIdx.x / (unsigned)rb);  // rb row blocks per graph
  const int st = d.status[g];
  if (st == PREDTOP_ERR_TOO_LARGE || st == PREDTOP_ERR_INVALID_ARG) return;
  const int64_t n0 = d.node_ptr[g];
  const int N = (int)(d.node_ptr[g + 1] - n0);
  if (is_small(N, (int)(d.edge_ptr[g + 1] - d.edge_ptr[g]), sc)) return;
  if (128 * a >= N) return;
  const int W = 2 * ((N + 127) / 128), T = (N + 127) / 128;
  const int rows = min(128, N - 128 * a);
  const uint64_t* Rg = d.R + d.row_off[g];
  uint64_t* Mg = d.M + d.row_off[g];
  int32_t* cnt = d.tile_cnt + d.tile_off[g] + (int64_t)a * T;
  const int tid = threadIdx.x, nt = blockDim.x, lane = tid & 31, warp = tid >> 5, nwarps = nt >> 5;
  if (st != PREDTOP_OK) {  // device-detected error: M defined as zero
    for (int64_t it = tid; it < (int64_t)rows * W; it += nt) Mg[(int64_t)(128 * a) * W + it] = 0;
    for (int t = tid; t < T; t += nt) cnt[t] = 0;
    return;
  }
  for (int t = tid; t < T; t += nt) s_cnt[t] = 0;
  for (int w0 = 0; w0 < W; w0 += kMC) {
    const int nw = min(kMC, W - w0);
    for (int it = tid; it < rows * nw; it += nt) {
      const int r = it / nw, c = it - r * nw;
      const uint64_t x = Rg[(int64_t)(128 * a + r) * W + w0 + c];
      sA[r * kMA + 2 * c] = (uint32_t)x;
      sA[r * kMA + 2 * c + 1] = (uint32_t)(x >> 32);
    }
    const int v0 = 64 * w0, nv = min(N, 64 * (w0 + nw)) - v0;
    for (int it = tid; it < 2 * nv; it += nt) {
      const int v = it >> 1, k = it & 1;
      const uint64_t x = Rg[(int64_t)(v0 + v) * W + 2 * a + k];
      sB[v * kMB + 2 * k] = (uint32_t)x;
      sB[v * kMB + 2 * k + 1] = (uint32_t)(x >> 32);
    }
    __syncthreads();
    // task (u sub-block us of 32 rows, v sub-block vs of 32 columns): lane i
    // of the transpose input holds strip row v0 + 32 vs + i (the bits of rows
    // u = 128a + 32us ..); on exit lane i holds the bits over v of row
    // u = 128a + 32us + i, i.e. 32-bit word vs of its chunk
    for (int task = warp; task < 4 * 2 * nw; task += nwarps) {
      const int us = task & 3, vs = task >> 2;
      const int vr = 32 * vs + lane;
      const uint32_t x = vr < nv ? sB[vr * kMB + us] : 0u;
      const uint32_t t = transpose32(x, lane);
      const int r = 32 * us + lane;
      if (r < rows) sA[r * kMA + vs] |= t;
    }
    __syncthreads();
    for (int it = tid; it < rows * nw; it += nt) {
      const int r = it / nw, c = it - r * nw;
      const int u = 128 * a + r, w = w0 + c;
      uint64_t m = ((uint64_t)sA[r * kMA + 2 * c + 1] << 32) | sA[r * kMA + 2 * c];
      if ((u >> 6) == w) m |= 1ull << (u & 63);
      Mg[(int64_t)u * W + w] = mask_perm(m);
      const int c1 = __popcll(m);
      if (c1) atomicAdd(&s_cnt[w >> 1], c1);
    }
    __syncthreads();
  }
  for (int t = tid; t < T; t += nt) cnt[t] = s_cnt[t];
}

__global__ void __launch_bounds__(256) k_classify(DagDev d, SmallCfg sc) {
  const int g = blockIdx.x;
  const int st = d.status[g];
  if (st == PREDTOP_ERR_TOO_LARGE || st == PREDTOP_ERR_INVALID_ARG) return;
  __shared__ unsigned long long s_pairs;
  const int N = (int)(d.node_ptr[g + 1] - d.node_ptr[g]);
  if (is_small(N, (int)(d.edge_ptr[g + 1] - d.edge_ptr[g]), sc)) return;
  const int T = (N + 127) / 128;
  const int32_t* cnt = d.tile_cnt + d.tile_off[g];
  uint8_t* cls = d.tile_cls + d.tile_off[g];
  if (threadIdx.x == 0) s_pairs = 0;
  __syncthreads();
  unsigned long long local = 0;
  for (int t = threadIdx.x; t < T * T; t += blockDim.x) {
    const int qt = t / T, kt = t % T;
    const int64_t cells = (int64_t)min(128, N - qt * 128) * min(128, N - kt * 128);
    const int c = cnt[t];
    cls[t] = (uint8_t)(c == 0 ? 0 : (c == cells ? 2 : 1));
    local += (unsigned long long)c;
  }
  atomicAdd(&s_pairs, local);  // integer: order-independent
  __syncthreads();
  if (threadIdx.x == 0) d.pairs[g] = (int64_t)s_pairs;
}


// ---------------------------------------------------------------------------
// Fused small-graph path: one warp per graph does K1 + K2 + K3 in shared
// memory (validation, successor CSR, Kahn depth, closure, mask, tile classes,
// |A|, attention work items) with __syncwarp between levels instead of CTA
// barriers.  GPT-size stage graphs (N ~ 300) need ~25 KB per warp.
__device__ __forceinline__ size_t small_int_bytes(const SmallCfg& sc) {
  return align_up((size_t)4 * (4 * (size_t)sc.sn + 2 + sc.se + 24), 16);
}

#ifdef PREDTOP_TRACE
// clock64 at the phase boundaries of k_dag_small, summed over graphs 0..63
__device__ long long g_dag_trace[8];
__device__ int g_dag_levels;
#define DTR(k)                                                      \
  do {                                                              \
    if (lane == 0 && g < 64) atomicAdd((unsigned long long*)&g_dag_trace[k], (unsigned long long)(clock64() - dt0)); \
  } while (0)
#else
#define DTR(k) \
  do {         \
  } while (0)
#endif

__global__ void __launch_bounds__(128) k_dag_small(DagDev d, int G, SmallCfg sc) {
  extern __shared__ __align__(16) unsigned char sm_small[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int g = blockIdx.x * 4 + warp;
  if (g >= G || d.status[g] != PREDTOP_OK) return;
  const int64_t n0 = d.node_ptr[g];
  const int N = (int)(d.node_ptr[g + 1] - n0);
  const int64_t e0 = d.edge_ptr[g];
  const int E = (int)(d.edge_ptr[g + 1] - e0);
  if (!is_small(N, E, sc)) return;
#ifdef PREDTOP_TRACE
  const long long dt0 = clock64();
#endif
  unsigned char* slot = sm_small + (size_t)warp * sc.slot;
  int* indeg = reinterpret_cast<int*>(slot);
  int* soff = indeg + sc.sn;        // N+1
  // E successors: shared slot when they fit, else the global CSR scratch
  int* succ = E <= sc.se ? soff + sc.sn + 1 : d.succ + e0;
  int* topo = soff + sc.sn + 1 + sc.se;  // N
  int* lptr = topo + sc.sn;         // N+1 (first the fill cursor)
  int* tcnt = lptr + sc.sn + 1;     // 16 tile counts (T <= 4)
  int* ctr = tcnt + 16;             // Kahn queue tail
  uint64_t* R = reinterpret_cast<uint64_t*>(slot + small_int_bytes(sc));
  const int W = 2 * ((N + 127) / 128), T = (N + 127) / 128;
  const int32_t* src = d.src + e0;
  const int32_t* dst = d.dst + e0;
  int32_t* depth = d.depth + n0;
  uint64_t* Rg = d.R + d.row_off[g];
  uint32_t* M32 = reinterpret_cast<uint32_t*>(d.M + d.row_off[g]);
  uint8_t* cls = d.tile_cls + d.tile_off[g];

  for (int v = lane; v < N; v += 32) { indeg[v] = 0; soff[v + 1] = 0; }
  if (lane < 16) tcnt[lane] = 0;
  if (lane == 0) { soff[0] = 0; *ctr = 0; }
  __syncwarp();
  bool rng = false, self = false;
  for (int e = lane; e < E; e += 32) {
    const int s = src[e], t = dst[e];
    if (s < 0 || s >= N || t < 0 || t >= N) rng = true;
    else if (s == t) self = true;
    else {
      atomicAdd(&indeg[t], 1);
      atomicAdd(&soff[s + 1], 1);
    }
  }
  rng = __any_sync(0xffffffffu, rng);
  self = __any_sync(0xffffffffu, self);
  int status = rng ? PREDTOP_ERR_RANGE : self ? PREDTOP_ERR_SELF_LOOP : PREDTOP_OK;
  __syncwarp();
  int level = 0;
  if (status == PREDTOP_OK) {
    int carry = 0;  // inclusive scan of out-degrees
    for (int base = 0; base < N; base += 32) {
      const int v = base + lane;
      int x = v < N ? soff[v + 1] : 0;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
      }
      if (v < N) soff[v + 1] = carry + x;
      carry += __shfl_sync(0xffffffffu, x, 31);
    }
    __syncwarp();
    for (int v = lane; v < N; v += 32) lptr[v] = soff[v];
    __syncwarp();
    for (int e = lane; e < E; e += 32) succ[atomicAdd(&lptr[src[e]], 1)] = dst[e];
    __syncwarp();
    DTR(0);
    // Kahn, level synchronous (P:137 depth = 1 + max predecessor depth)
    int tail = 0;
    for (int base = 0; base < N; base += 32) {
      const int v = base + lane;
      const bool z = v < N && indeg[v] == 0;
      const uint32_t bal = __ballot_sync(0xffffffffu, z);
      if (z) {
        topo[tail + __popc(bal & ((1u << lane) - 1u))] = v;
        depth[v] = 0;
      }
      tail += __popc(bal);
    }
    if (lane == 0) lptr[0] = 0;
    __syncwarp();
    // frontier topo[lb, le); the warp-uniform tail needs no atomics: the
    // nodes a level releases are appended by ballot + prefix popcount
    const uint32_t lt = (1u << lane) - 1u;
    int lb = 0, le = tail;
    while (lb < le) {
      for (int i0 = lb; i0 < le; i0 += 32) {
        int k = 0, kend = 0;
        if (i0 + lane < le) {
          const int v = topo[i0 + lane];
          k = soff[v];
          kend = soff[v + 1];
        }
        while (__any_sync(0xffffffffu, k < kend)) {
          int w = 0;
          bool ready = false;
          if (k < kend) {
            w = succ[k++];
            ready = atomicSub(&indeg[w], 1) == 1;
          }
          const uint32_t bal = __ballot_sync(0xffffffffu, ready);
          if (ready) {
            topo[tail + __popc(bal & lt)] = w;
            depth[w] = level + 1;
          }
          tail += __popc(bal);
        }
      }
      __syncwarp();
      lb = le;
      le = tail;
      ++level;
      if (lane == 0) lptr[level] = lb;
    }
    __syncwarp();
    if (le != N) status = PREDTOP_ERR_CYCLE;
    DTR(1);
#ifdef PREDTOP_TRACE
    if (lane == 0 && g < 64) atomicAdd(&g_dag_levels, level);
#endif
  }
  if (lane == 0) d.num_levels[g] = level;
  if (status != PREDTOP_OK) {
    if (lane == 0) {
      d.status[g] = status;
      atomicMin(d.first_bad, g);
    }
    for (int v = lane; v < N; v += 32) depth[v] = -1;
    for (int64_t i = lane; i < (int64_t)N * W; i += 32) Rg[i] = 0;
    for (int64_t i = lane; i < (int64_t)N * 2 * W; i += 32) M32[i] = 0;
    for (int t = lane; t < T * T; t += 32) cls[t] = 0;
    return;
  }
  const int K = d.hops;
  if (K > 0 && K < level - 1) {
    // finite-k DAGRA: K synchronous rounds R_j[v] = OR_{w in
    // succ(v)} ({w} | R_{j-1}[w]), R_0 = 0, ping-ponging between the shared
    // slot and the graph's global R rows (rewritten from the slot below);
    // round j writes the slot iff K - j is even, so R_K ends in the slot.
    // (K >= longest path = level - 1 gives the full closure: path below.)
    for (int j = 1; j <= K; ++j) {
      const bool to_smem = ((K - j) & 1) == 0;
      uint64_t* dstb = to_smem ? R : Rg;
      const uint64_t* srcb = to_smem ? Rg : R;
      for (int it = lane; it < N * W; it += 32) {
        const int v = it / W, c = it % W;
        uint64_t acc = 0;
        for (int k = soff[v]; k < soff[v + 1]; ++k) {
          const int w = succ[k];
          if (j > 1) acc |= to_smem ? __ldcg(srcb + w * W + c) : srcb[w * W + c];
          if ((w >> 6) == c) acc |= 1ull << (w & 63);
        }
        dstb[it] = acc;
      }
      __threadfence();
      __syncwarp();
    }
  } else {
  // closure R[v] = OR_{w in succ(v)} (R[w] | {w}), deepest level first.
  // Per topo position a packed record replaces the topo -> soff -> succ load
  // chain of the latency-bound level loop: lo = v | deg << 9 | s0 << 12 |
  // s1 << 21 (in topo[]), hi = s2 | s3 << 9 | s4 << 18 (in indeg[], dead
  // after Kahn); node ids < 512 fit 9 bits; deg > 5 is marked 7 and read
  // from the CSR.
  for (int i = lane; i < N; i += 32) {
    const int v = topo[i], b = soff[v], deg = soff[v + 1] - b;
    int sv[5] = {0, 0, 0, 0, 0};
#pragma unroll
    for (int k = 0; k < 5; ++k)
      if (k < deg) sv[k] = succ[b + k];
    topo[i] = v | (min(deg, 6) == 6 ? 7 << 9 : deg << 9) | (sv[0] << 12) | (sv[1] << 21);
    indeg[i] = sv[2] | (sv[3] << 9) | (sv[4] << 18);
  }
  for (int i = lane; i < N * W; i += 32) R[i] = 0;
  __syncwarp();
  const int ln = lane / W, lw = lane - (lane / W) * W;  // this lane's first item of a level
  for (int l = level - 1; l >= 0; --l) {
    const int lb = lptr[l], items = (lptr[l + 1] - lb) * W;
    for (int it = lane; it < items; it += 32) {
      int ni = ln, j = lw;
      if (it != lane) {
        ni = it / W;
        j = it - ni * W;
      }
      const uint32_t lo = (uint32_t)topo[lb + ni], hi = (uint32_t)indeg[lb + ni];
      const int v = (int)(lo & 511u), degc = (int)((lo >> 9) & 7u);
      uint64_t acc = 0;
      if (degc <= 5) {
        const int sv[5] = {(int)((lo >> 12) & 511u), (int)((lo >> 21) & 511u), (int)(hi & 511u),
                           (int)((hi >> 9) & 511u), (int)((hi >> 18) & 511u)};
#pragma unroll
        for (int k = 0; k < 5; ++k)
          if (k < degc) {
            const int w = sv[k];
            acc |= R[w * W + j] | ((w >> 6) == j ? 1ull << (w & 63) : 0ull);
          }
      } else {
        for (int k = soff[v]; k < soff[v + 1]; ++k) {
          const int w = succ[k];
          acc |= R[w * W + j];
          if ((w >> 6) == j) acc |= 1ull << (w & 63);
        }
      }
      R[v * W + j] = acc;
    }
    __syncwarp();
  }
  }
  DTR(2);
  // mask M = R | R^T | I per 64-bit word (two 32x32 bit transposes in
  // flight), written in the stored layout (mask_perm); R written out in the
  // same pass; per-tile popcounts
  const uint32_t* R32 = reinterpret_cast<const uint32_t*>(R);
  const int W32 = 2 * W, NB = (N + 31) / 32;
  uint64_t* Mw = d.M + d.row_off[g];
  for (int ur = 0; ur < NB; ++ur) {
    const int U0 = ur * 32, u = U0 + lane;
    int ctile[4] = {0, 0, 0, 0};  // this lane's popcounts per 128-key tile (W <= 8)
    for (int vw = 0; vw < W; ++vw) {
      const int V0 = vw * 64;
      const uint32_t dlo = u < N ? R32[u * W32 + 2 * vw] : 0u;
      const uint32_t dhi = u < N ? R32[u * W32 + 2 * vw + 1] : 0u;
      const uint32_t xlo = V0 + lane < N ? R32[(V0 + lane) * W32 + ur] : 0u;
      const uint32_t xhi = V0 + 32 + lane < N ? R32[(V0 + 32 + lane) * W32 + ur] : 0u;
      const uint32_t tlo = transpose32(xlo, lane), thi = transpose32(xhi, lane);
      if (u < N) Rg[(int64_t)u * W + vw] = ((uint64_t)dhi << 32) | dlo;
      uint32_t mlo = dlo | tlo, mhi = dhi | thi;
      if (U0 == V0) mlo |= 1u << lane;
      if (U0 == V0 + 32) mhi |= 1u << lane;
      if (u >= N) mlo = mhi = 0u;
      if (u < N) Mw[(int64_t)u * W + vw] = mask_perm(((uint64_t)mhi << 32) | mlo);
      const int c = __popc(mlo) + __popc(mhi);
#pragma unroll
      for (int tt = 0; tt < 4; ++tt)
        if (tt == vw / 2) ctile[tt] += c;
    }
#pragma unroll
    for (int tt = 0; tt < 4; ++tt) {
      int c = ctile[tt];
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
      if (lane == 0 && tt < T) tcnt[(U0 / 128) * T + tt] += c;
    }
  }
  __syncwarp();
  DTR(3);
  long long pairs = 0;
  for (int t = lane; t < T * T; t += 32) {
    const int qt = t / T, kt = t % T;
    const int cells = min(128, N - qt * 128) * min(128, N - kt * 128);
    const int c = tcnt[t];
    cls[t] = (uint8_t)(c == 0 ? 0 : (c == cells ? 2 : 1));
    pairs += c;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) pairs += __shfl_xor_sync(0xffffffffu, pairs, o);
  if (lane == 0) d.pairs[g] = pairs;
  DTR(4);
}

// Block flags for the attention kernel: for every 16-row group rg and 64-key
// chunk c, bit j (j < 4) = some row of the group has an allowed key in the
// permuted 16-key block j (mask bits 0x000F000F000F000F << 4j, attention.cu),
// bit 4+j = every row of the group allows every key of block j.
__global__ void __launch_bounds__(128) k_bflags(DagDev d, SmallCfg sc) {
  const int g = blockIdx.x;
  if (d.status[g] == PREDTOP_ERR_TOO_LARGE || d.status[g] == PREDTOP_ERR_INVALID_ARG) return;
  const int N = (int)(d.node_ptr[g + 1] - d.node_ptr[g]);
  // k_dag_small and k_mask2 write M in the stored layout already
  (void)sc;
  const int W = 2 * ((N + 127) / 128), nch = (N + 63) / 64, ng = (N + 15) / 16;
  const uint64_t* Mg = d.M + d.row_off[g];
  uint8_t* out = d.bflag + d.bflag_off[g];
  // grid (G, Y): the (16-row group, chunk) items of a graph are spread over
  // gridDim.y CTAs, so one large graph (16k nodes: 262k items) is not a
  // single-CTA loop
  for (int it = blockIdx.y * blockDim.x + threadIdx.x; it < ng * nch; it += gridDim.y * blockDim.x) {
    const int rg = it / nch, c = it % nch;
    uint64_t o = 0, a = ~0ull;
    for (int r = rg * 16; r < min(N, rg * 16 + 16); ++r) {
      const uint64_t w = Mg[(int64_t)r * W + c];
      o |= w;
      a &= w;
    }
    uint32_t f = 0;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const uint64_t MJ = 0x000F000F000F000Full << (4 * j);
      if (o & MJ) f |= 1u << j;
      if ((a & MJ) == MJ) f |= 16u << j;
    }
    out[it] = (uint8_t)f;
  }
}

__global__ void k_copy_words(const int64_t* total, const uint64_t* from, uint64_t* to, bool unperm) {
  const int64_t n = *total;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    to[i] = unperm ? mask_unperm(from[i]) : from[i];
}

predtop_status dag_build_launch(predtop_dag_s* dag, cudaStream_t st) {
  const predtop_batch_desc& b = dag->desc;
  const DagDev& d = dag->d;
  const int G = b.num_graphs;
  // small-graph capacity: graphs up to 512 nodes run fused (k_dag_small);
  // when the batch's max_nodes is within it, the multi-kernel path is not
  // launched at all
  SmallCfg sc{0, 0, 0};
  if (b.max_nodes <= 512) {
    sc.sn = b.max_nodes;
    sc.se = 4 * b.max_nodes;
    const size_t ib = align_up((size_t)4 * (4 * (size_t)sc.sn + 2 + sc.se + 24), 16);
    sc.slot = (int)align_up(ib + (size_t)sc.sn * 2 * ceil_div(sc.sn, 128) * 8, 16);
  }
  const bool all_small = sc.sn > 0;
  if (!all_small)
    PT_CUDA_TRY(cudaMemsetAsync(d.tile_cnt, 0, sizeof(int32_t) * (size_t)dag->tiles_bound, st));
{
    ProfScope _p(PK_DAG_META, st);
    k_meta<<<1, 1024, 0, st>>>(d, G, b.max_nodes);
    PT_LAUNCH_CHECK();
  }
  if (all_small) {
    PT_SMEM_ATTR(k_dag_small, 4 * sc.slot);
    ProfScope _p(PK_DAG_SMALL, st);
    k_dag_small<<<(unsigned)ceil_div(G, 4), 128, 4 * sc.slot, st>>>(d, G, sc);
    PT_LAUNCH_CHECK();
  } else {
{
    // in-degrees and the Kahn queue in shared memory when the largest graph
    // fits; warp mode (16-bit CSR in shared memory too) for graphs with at
    // most `ecap` edges: 8 N + 2 + 2 ecap bytes, ecap <= 4 N within 200 KB
    const int smem_nodes = b.max_nodes <= 24 * 1024 ? b.max_nodes : 0;
    int ecap = 0;
    if (smem_nodes > 0)
      ecap = (int)std::min<int64_t>(4 * (int64_t)smem_nodes, (200 * 1024 - 8 * (int64_t)smem_nodes - 2) / 2);
    const int dsm = (int)align_up((size_t)8 * smem_nodes + 2 + 2 * (size_t)std::max(ecap, 0), 16);
    PT_SMEM_ATTR(k_depth, dsm);
    ProfScope _p(PK_DAG_DEPTH, st);
    k_depth<<<G, 256, dsm, st>>>(d, sc, smem_nodes, std::max(ecap, 0));
    PT_LAUNCH_CHECK();
  }
  const int64_t maxN = b.max_nodes;
  const int64_t Wmax = dag->max_words;
  if (b.hops == 0 && maxN > kDeepNodes) {
    // deep graphs: 16-bit column chains, `cpb` per CTA, one CTA per SM
    const int cpb = (int)std::max<int64_t>(1, std::min<int64_t>(8, (227 * 1024 - 64) / (2 * maxN)));
    const int csm = (int)align_up((size_t)cpb * 2 * (size_t)maxN, 16);
    PT_SMEM_ATTR(k_closure16, csm);
    ProfScope _p(PK_DAG_CLOSURE, st);
    k_closure16<<<dim3(G, (unsigned)ceil_div(4 * Wmax, cpb)), 256, csm, st>>>(d, sc, cpb);
    PT_LAUNCH_CHECK();
  } else {
  // closure: shared memory for a column slice of all rows of the largest graph
  // (+ its CSR when it fits); several CTAs per SM for small graphs.
  int64_t want = maxN * Wmax * 8 + 4 * (4 * maxN + 8) + 16;  // R slice + CSR (E ~ 2N)
  int smem = (int)std::min<int64_t>(want, 200 * 1024);
  smem = (int)align_up((size_t)smem, 1024);
  PT_SMEM_ATTR(k_closure, 200 * 1024);
  int64_t cw = std::max<int64_t>(1, std::min<int64_t>(Wmax, (int64_t)smem / (8 * maxN)));
  int64_t slices = ceil_div(Wmax, cw);
  if ((int64_t)smem < 8 * maxN) slices = std::min<int64_t>(ceil_div(Wmax, 2), 65535);  // global mode
  dim3 gc(G, (unsigned)std::max<int64_t>(1, slices));
{
    ProfScope _p(PK_DAG_CLOSURE, st);
    k_closure<<<gc, 256, smem, st>>>(d, smem, sc);
    PT_LAUNCH_CHECK();
  }
  }
{
    ProfScope _p(PK_DAG_MASK, st);
    PT_SMEM_ATTR(k_mask2, (int)kMaskSmem);
    // 1D grid of G x rb CTAs, the row blocks of a graph consecutive
    const int64_t rb = ceil_div(maxN, 128);
    if ((int64_t)G * rb > 0x7fffffff) {
      set_error("mask grid too large");
      return PREDTOP_ERR_TOO_LARGE;
    }
    k_mask2<<<(unsigned)(G * rb), 256, kMaskSmem, st>>>(d, sc, (int)rb);
    PT_LAUNCH_CHECK();
  }
{
    ProfScope _p(PK_DAG_CLASSIFY, st);
    k_classify<<<G, 256, 0, st>>>(d, sc);
    PT_LAUNCH_CHECK();
  }
  }  // multi-kernel path
  {
    ProfScope _p(PK_DAG_FLAGS, st);
    const int64_t items = ceil_div(b.max_nodes, 16) * ceil_div(b.max_nodes, 64);
    dim3 gb(G, (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(items, 128), 1024)));
    k_bflags<<<gb, 128, 0, st>>>(d, sc);
    PT_LAUNCH_CHECK();
  }
  return PREDTOP_OK;
}

predtop_status dag_copy_bits(const predtop_dag_s* dag, const uint64_t* from, uint64_t* to,
                             cudaStream_t st, bool unperm) {
  const int G = dag->desc.num_graphs;
{
    ProfScope _p(PK_COPY, st);
    k_copy_words<<<592, 256, 0, st>>>(dag->d.row_off + G, from, to, unperm);
    PT_LAUNCH_CHECK();
  }
  return PREDTOP_OK;
}

}  // namespace predtop

#ifdef PREDTOP_TRACE
extern "C" PREDTOP_API int predtop_debug_dag_trace(long long* out) {
  if (cudaMemcpyFromSymbol(out, predtop::g_dag_trace, sizeof(predtop::g_dag_trace)) != cudaSuccess) return -7;
  return cudaMemcpyFromSymbol(out + 8, predtop::g_dag_levels, sizeof(int)) == cudaSuccess ? 0 : -7;
}
#endif
