// internal.h -- handle structs and launcher prototypes shared by the .cu files
// of libpredtop.  Not part of the ABI.
#pragma once
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <vector>

#include "common.cuh"

namespace predtop {

// Device views of a built batch of stage DAGs (all carved from the caller's
// build_dag workspace, except the borrowed input arrays).
struct DagDev {
  // borrowed inputs
  const int64_t* node_ptr;
  const int64_t* edge_ptr;
  const int32_t* src;
  const int32_t* dst;
  const predtop_node_feat* feats;
  // per graph
  int32_t* status;     // [G]   predtop_status of the graph
  int32_t* num_levels; // [G]
  int64_t* row_off;    // [G+1] word offset of the graph's bitset rows (prefix of N_g*W_g)
  int64_t* tile_off;   // [G+1] prefix of T_g^2
  int32_t* qtile_off;  // [G+1] prefix of T_g (attention work items)
  int64_t* pairs;      // [G]   |A_g|
  int32_t* first_bad;  // [1]   lowest bad graph (INT_MAX if none)
  // per node / edge
  int32_t* depth;      // [N_tot] caller order
  int32_t* topo;       // [N_tot] graph-local ids by level
  int32_t* level_ptr;  // [N_tot + G] graph g at node_ptr[g] + g
  int32_t* succ_off;   // [N_tot + G] graph g at node_ptr[g] + g
  int32_t* succ;       // [E]  graph-local successor lists
  int32_t* indeg;      // [N_tot]
  int4* rec;           // [N_tot] per topo position: {v | deg << 16, s0 | s1 << 16, s2 | s3 << 16, soff[v]}
                       // (the first four successors inline; large-graph closure)
  // bitsets and tiles
  uint64_t* R;         // [sum N_g W_g]
  uint64_t* M;         // [sum N_g W_g]  STORED layout: mask_perm of each 64-key word
  int32_t* tile_cnt;   // [sum T_g^2]
  uint8_t* tile_cls;   // [sum T_g^2]
  int2* work;          // [qtile bound] (graph, q-tile) attention work items
  int64_t* bflag_off;  // [G+1] prefix of ceil(N/16) * ceil(N/64)
  uint8_t* bflag;      // per (16-row group, 64-key chunk): bits 0-3 block (keys 16j..16j+15)
                       // has an allowed pair, bits 4-7 block fully allowed (attention.cu)
  int32_t hops;        // DAGRA range k (0 = infinity): R is then the k-hop relation R_k
};

// Stored layout of the attention mask words.  Key k (0..63) of a 64-key chunk
// sits at bit mask_pos(k) = 16*((k>>1)&3) + 2*(k>>3) + (k&1): in the m16n8
// accumulator fragment of the QK^T MMA, thread tq (= lane%4) holds for n-tile
// nt (8 keys) the keys 8nt + 2tq + {0,1}, so its 16 keys of the chunk are the
// contiguous bits [16tq, 16tq+16), ordered (nt, u), and 16-key block j is
// 0x000F000F000F000F << 4j.  k_bflags converts the natural-order words the
// mask kernels write; predtop_debug_mask converts back.
__host__ __device__ constexpr int mask_pos(int k) { return 16 * ((k >> 1) & 3) + 2 * (k >> 3) + (k & 1); }
__device__ __forceinline__ uint64_t mask_perm(uint64_t w) {  // natural -> stored
  uint64_t out = 0;
#pragma unroll
  for (int tq = 0; tq < 4; ++tq) {  // bits (2tq, 2tq+1) of every byte -> 16-bit field tq
    uint64_t x = (w >> (2 * tq)) & 0x0303030303030303ull;
    x = (x | (x >> 6)) & 0x000F000F000F000Full;
    x = (x | (x >> 12)) & 0x000000FF000000FFull;
    x = (x | (x >> 24)) & 0xFFFFull;
    out |= x << (16 * tq);
  }
  return out;
}
__device__ __forceinline__ uint64_t mask_unperm(uint64_t w) {  // stored -> natural
  uint64_t out = 0;
#pragma unroll
  for (int tq = 0; tq < 4; ++tq) {
    uint64_t x = (w >> (16 * tq)) & 0xFFFFull;
    x = (x | (x << 24)) & 0x000000FF000000FFull;
    x = (x | (x << 12)) & 0x000F000F000F000Full;
    x = (x | (x << 6)) & 0x0303030303030303ull;
    out |= x << (2 * tq);
  }
  return out;
}

}  // namespace predtop

struct predtop_dag_s {
  predtop_batch_desc desc;
  predtop::DagDev d;
  int64_t words_bound;  // upper bound of sum N_g W_g
  int64_t tiles_bound;  // upper bound of sum T_g^2
  int64_t qtiles_bound; // upper bound of sum T_g
  int64_t bflags_bound; // upper bound of sum ceil(N/16) ceil(N/64)
  int32_t max_words;    // 2*ceil(max_nodes/128)
};

namespace predtop {

constexpr int kMaxLayers = 16;

struct LayerDev {
  __half* Wqkv;  // [3d][d]
  float* bqkv;   // [3d]
  __half* Wo;    // [d][d]
  float* bo;
  float* g1;
  float* be1;
  __half* W1;    // [dff][d]
  float* b1;
  __half* W2;    // [d][dff]
  float* b2;
  float* g2;
  float* be2;
  CUtensorMap tm_qkv, tm_o, tm_1, tm_2;  // B-operand TMA maps (unfused GEMMs)
  CUtensorMap tm_1c;                     // W_1 in 128-row chunks (fused layer tail v1)
  CUtensorMap tm_1h;                     // W_1 in 64-row chunks (layer tail v2)
  CUtensorMap tm_o32, tm_2_32;           // W_o, W_2 in 32-wide K-slices (LN GEMMs at d = 256)
};

}  // namespace predtop

struct predtop_model_s {
  predtop_model_config cfg;
  float* W_inT;  // [F][d] (transposed: one-hot rows are gathers)
  float* b_in;   // [d]
  predtop::LayerDev layer[predtop::kMaxLayers];
  float* H1T;    // [d][d] transposed (in-major)
  float* c1;
  float* H2T;
  float* c2;
  float* w_o;    // [d]
  float* c_o;    // [1]
  int bn_qkv, bn_ff1;  // GEMM N-tile widths
};

namespace predtop {

// ---- dag.cu
predtop_status dag_build_launch(predtop_dag_s* dag, cudaStream_t st);
predtop_status dag_copy_bits(const predtop_dag_s* dag, const uint64_t* from, uint64_t* to,
                             cudaStream_t st, bool unperm = false);

// ---- tma.cu
bool encode_tma_2d(CUtensorMap* map, const void* base, int elem_bytes, uint64_t inner,
                   uint64_t outer, uint32_t box_inner, uint32_t box_outer);
bool encode_tma_2d_f16(CUtensorMap* map, const void* base, uint64_t inner, uint64_t outer,
                       uint32_t box_inner, uint32_t box_outer);

// ---- gemm.cu
enum GemmEpi { EPI_BIAS_F16 = 0, EPI_BIAS_RELU_F16 = 1, EPI_BIAS_RESID_LN = 2 };
struct GemmArgs {
  int M, K, N;           // rows, reduction, total output columns
  const float* bias;     // [N]
  __half* out16;         // [M][N]
  float* out32;          // [M][N]   (LN epilogue)
  const float* resid32;  // [M][N]   (LN epilogue; may alias out32)
  const float* gamma;
  const float* beta;
  float eps;
  int qcols;      // bias epilogue: output columns [0, qcols) are multiplied by qscale
  float qscale;   // (QKV: Q pre-scaled by log2(e)/sqrt(d_h) for the attention kernel)
  int kch;        // K-slice of the operand maps (0: 64 if K % 64 == 0, else 32)
};
predtop_status gemm_launch(const CUtensorMap* tmA, const CUtensorMap* tmB, int bn, int epi,
                           const GemmArgs& a, cudaStream_t st);
int gemm_pick_bn(int N);

// ---- embed.cu / readout.cu / attention.cu / plan.cu
predtop_status pe_table_launch(float* pe, int max_depth, int d, cudaStream_t st);
predtop_status embed_launch(const predtop_model_s* m, const predtop_dag_s* dag, const float* pe,
                            float* x32, __half* x16, cudaStream_t st);
bool attention_tc_supported(const predtop_dag_s* dag, int d, int H);
// graphs with at least nmin nodes (0: all)
predtop_status attention_tc_launch(const predtop_dag_s* dag, int d, int H, const __half* qkv, __half* out,
                                   cudaStream_t st, int nmin = 0);
predtop_status attention_launch(const predtop_dag_s* dag, int d, int H, const __half* qkv,
                                __half* out, cudaStream_t st);
predtop_status readout_launch(const predtop_model_s* m, const predtop_dag_s* dag, const float* x32,
                              float* latency, cudaStream_t st);
predtop_status plan_launch(int64_t P, const int64_t* plan_ptr, const int32_t* plan_stage,
                           const int32_t* B, const float* t, int64_t num_stages, double* T,
                           int64_t* first_bad, cudaStream_t st);
predtop_status argmin_launch(int64_t n, const double* T, int64_t* best, cudaStream_t st);

// ---- prune.cu (graph pruning)
size_t prune_workspace_bytes(const predtop_batch_desc* b);
predtop_status prune_launch(const predtop_batch_desc* b, const int64_t* node_ptr, const int64_t* edge_ptr,
                            const int32_t* src, const int32_t* dst, const predtop_node_feat* feats,
                            const uint16_t* ops, int n_ops, void* ws, int64_t* out_node_ptr,
                            int64_t* out_edge_ptr, int32_t* out_src, int32_t* out_dst,
                            int64_t edge_capacity, predtop_node_feat* out_feats, int64_t* totals_host,
                            int32_t* first_bad_host, cudaStream_t st);

// ---- search.cu (inter-stage plan search)
size_t search_workspace_bytes(int64_t P, int L, int K);  // [P][K * L(L+1)/2] candidate T
predtop_status search_launch(int64_t P, int L, int K, const int32_t* dev, int D, const float* t,
                             int64_t stride, int64_t num_tables, const int32_t* table_of, const int32_t* B,
                             double* T_out, int32_t* S_out, int32_t* end_out, int32_t* choice_out,
                             void* ws, cudaStream_t st);

// ---- layer.cu (fused O-proj + LN1 + FFN + LN2)
bool layer_tail_supported(int d, int dff);
bool layer_tail2_supported(int d, int dff);
predtop_status layer_tail2_launch(const predtop_model_s* m, int l, const __half* att, float* x32,
                                  __half* x16, int M, cudaStream_t st);
predtop_status layer_tail_launch(const predtop_model_s* m, int l, const __half* att, float* x32,
                                 __half* x16, int M, cudaStream_t st);

// ---- layer256.cu (fused O-proj + LN1 + FFN + LN2 at d = 256)
bool layer_tail256_supported(int d, int dff);
predtop_status layer_tail256_launch(const predtop_model_s* m, int l, const __half* att, float* x32,
                                    __half* x16, int M, cudaStream_t st);

}  // namespace predtop
