/*
 * predtop.h -- C ABI of libpredtop, the B200 (sm_100a) implementation of the
 * prediction phase of PredTOP (Acharya & Shu, IPDPS 2025).
 *
 * Citations "P:n" refer to line n of the paper text, with the
 * section / equation / table named beside it.
 *
 * The prediction phase (SVI-3): "use the DAG Transformer model
 * trained in the previous phase to make predictions for the runtime latency
 * of all the stages on the corresponding mesh ... we use the pipeline model to
 * get the end-to-end latency of the DL training iteration."  The library
 * exposes that path as four calls:
 *
 *   predtop_build_dag      stage DAGs (SIV-B2) -> validated, depth
 *                          (DAGPE) and reachability closure (DAGRA,
 *                          P:135/P:145 with k = infinity) in device workspace
 *   predtop_reachability   export the closure bitsets (caller order)
 *   predtop_stage_forward  DAG-Transformer forward (Eqn 1 P:140-142, layers
 *                          P:172, global add pool Eqn 2 P:174, MLP head P:176)
 *                          -> one fp32 latency per stage graph
 *   predtop_plan_latency   white-box pipeline model, Eqn 4:
 *                          T = sum_i t_i + (B - 1) * max_j t_j
 *
 * Conventions that hold for every call:
 *  - Status: every call returns predtop_status (0 = ok, < 0 = error) and never
 *    throws, aborts or exits across the ABI.  predtop_last_error() returns a
 *    thread-local human-readable message for the last failing call.
 *  - Memory: the CALLER owns all device memory (inputs, outputs, workspaces,
 *    model weights).  The library never calls cudaMalloc/cudaFree.  Handles
 *    (predtop_dag, predtop_model) are small host structs that point into
 *    caller memory; the caller keeps that memory alive until *_destroy.
 *  - Pointers: array arguments are DEVICE pointers unless marked [host].
 *    All device work is stream-ordered on `cuda_stream` (a cudaStream_t,
 *    NULL = legacy default stream).  Input arrays are only read during the
 *    call's stream-ordered work, except that a predtop_dag keeps node_ptr,
 *    edge_ptr and feats (and depth_out) by reference for the later
 *    predtop_stage_forward calls on it.
 *  - CUDA graphs: with PREDTOP_NO_SYNC every call is stream-capturable (no
 *    host synchronisation, no allocation), so a whole prediction step can be
 *    captured once and replayed (bench.py does).
 *  - There is no CPU fallback: without a usable sm_100 device every call that
 *    launches work returns PREDTOP_ERR_CUDA.
 */
#ifndef PREDTOP_H
#define PREDTOP_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define PREDTOP_API __attribute__((visibility("default")))
#else
#define PREDTOP_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

#define PREDTOP_ABI_VERSION 2 /* 2: predtop_batch_desc.hops */

typedef enum {
  PREDTOP_OK = 0,
  PREDTOP_ERR_INVALID_ARG = -1, /* null pointer, bad size, bad config, bad plan */
  PREDTOP_ERR_RANGE = -2,       /* an edge endpoint outside [0, N_g) */
  PREDTOP_ERR_SELF_LOOP = -3,   /* an edge u -> u */
  PREDTOP_ERR_CYCLE = -4,       /* the graph is not acyclic ("DAG") */
  PREDTOP_ERR_TOO_LARGE = -5,   /* N_g > PREDTOP_MAX_NODES, or sizes overflow */
  PREDTOP_ERR_WORKSPACE = -6,   /* workspace too small or misaligned */
  PREDTOP_ERR_CUDA = -7,        /* CUDA error / no sm_100 device */
  PREDTOP_ERR_UNSUPPORTED = -8  /* a model shape the kernels do not support */
} predtop_status;

/* ---------------------------------------------------------------------------
 * Node features: Table I and SIV-B3.
 *   operator type    -> one-hot of `op`      (PREDTOP_NUM_OPS slots)
 *   output dims      -> ln(1 + dims[j]), "logarithmic scaling";
 *                       rank < 4 is zero-padded (ln(1+0) = 0)
 *   output data type -> one-hot of `dtype`   (PREDTOP_NUM_DTYPES slots)
 *   node type        -> one-hot of `kind`: input, literal, operator, output
 * The dense feature vector f(v) (length PREDTOP_NUM_FEATURES) is, in order:
 *   [ onehot(op) | ln(1+dims[0..3]) | onehot(dtype) | onehot(kind) ]
 * The record crosses the ABI in this compact 20-byte form; the one-hot part
 * is expanded on the device as a row gather.
 * ------------------------------------------------------------------------- */
#define PREDTOP_NUM_OPS 64
#define PREDTOP_NUM_DIMS 4
#define PREDTOP_NUM_DTYPES 8
#define PREDTOP_NUM_KINDS 4
#define PREDTOP_NUM_FEATURES \
  (PREDTOP_NUM_OPS + PREDTOP_NUM_DIMS + PREDTOP_NUM_DTYPES + PREDTOP_NUM_KINDS)

enum { PREDTOP_KIND_INPUT = 0, PREDTOP_KIND_LITERAL = 1,
       PREDTOP_KIND_OPERATOR = 2, PREDTOP_KIND_OUTPUT = 3 };

typedef struct {
  uint16_t op;      /* 0 .. PREDTOP_NUM_OPS-1 (values >= are clamped out: feature row all-zero) */
  uint8_t dtype;    /* 0 .. PREDTOP_NUM_DTYPES-1 (same rule) */
  uint8_t kind;     /* 0 .. PREDTOP_NUM_KINDS-1 (same rule) */
  uint32_t dims[4]; /* output tensor dims, zero-padded */
} predtop_node_feat;  /* 20 bytes, 4-byte aligned */

/* ---------------------------------------------------------------------------
 * A batch of stage DAGs (D1), packed:
 *   graph g owns nodes  [node_ptr[g], node_ptr[g+1])   N_g = node_ptr[g+1]-node_ptr[g]
 *   graph g owns edges  [edge_ptr[g], edge_ptr[g+1])
 *   edge e of graph g is edge_src[e] -> edge_dst[e] ("data dependency"),
 *   in GRAPH-LOCAL node ids 0..N_g-1.  Node order is arbitrary (any relabelling);
 *   every per-node output is in the caller's order.  Duplicate edges and
 *   isolated nodes are allowed.
 * ------------------------------------------------------------------------- */
#define PREDTOP_MAX_NODES 65536 /* per graph: the bitset closure is N^2/8 bytes */

enum { PREDTOP_NO_SYNC = 1u }; /* flags: do not synchronise to report device-detected errors */

typedef struct {
  int32_t num_graphs;   /* G >= 1 */
  int32_t max_nodes;    /* >= max_g N_g (an upper bound is fine; sizes workspaces) */
  int64_t total_nodes;  /* = node_ptr[G] */
  int64_t total_edges;  /* = edge_ptr[G] */
  uint32_t flags;       /* PREDTOP_NO_SYNC or 0 */
  int32_t hops;         /* DAGRA range k (Eqn 1 "u in N_k(v)" P:142; "the constant k ...
                           specifies the neighborhood range" P:145): 0 = k = infinity
                           (the paper's setting, full closure); k >= 1 = the k-hop
                           relation R_k below.  < 0 -> INVALID_ARG.  Occupies what was
                           tail padding: a zero-initialised ABI-v1 descriptor means k = inf. */
} predtop_batch_desc;

typedef struct predtop_dag_s* predtop_dag;
typedef struct predtop_model_s* predtop_model;

/* Bytes of device workspace predtop_build_dag needs for `desc` (256-byte
 * aligned base required).  0 on invalid desc. */
PREDTOP_API size_t predtop_build_dag_workspace(const predtop_batch_desc* desc);

/* Validate every graph, compute node depth and the reachability closure.
 *  - Validation, in this precedence per graph: RANGE (an endpoint outside
 *    [0,N_g)), SELF_LOOP, CYCLE (the stage graph is a DAG).  Also
 *    N_g < 1 or N_g > min(max_nodes, PREDTOP_MAX_NODES) -> TOO_LARGE.
 *  - depth (DAGPE): depth(v) = 0 if v has no predecessor, else
 *    1 + max over predecessors p of depth(p)  (longest path from a source).
 *  - reachability (DAGRA, P:135, P:145 with k = infinity): R[v] = the set of
 *    nodes u != v reachable from v by a directed path of >= 1 edge.
 *    With desc->hops = k >= 1 (finite-k DAGRA; R19):
 *    R_k[v] = the nodes u != v whose shortest directed path from v has at
 *    most k edges; predtop_reachability, the mask and stage_forward then use
 *    R_k (M = R_k | R_k^T | I).  k >= the longest path gives R exactly.
 *    The attention mask used by stage_forward is M = R | R^T | I
 *    ("a path from m to n or vice versa"; reflexive).
 * Arguments:
 *  node_ptr[G+1], edge_ptr[G+1]   int64, device
 *  edge_src[E], edge_dst[E]       int32, device, graph-local ids
 *  feats[N_tot]                   device; kept by reference in the handle and
 *                                 read again by predtop_stage_forward, so it
 *                                 must stay alive and unchanged until then
 *  workspace/ws_bytes             device, >= predtop_build_dag_workspace(desc)
 *  depth_out[N_tot]               int32 device, nullable
 *  out                            [host] receives the handle (valid even on a
 *                                 device-detected error; destroy it)
 *  first_bad_graph                [host] nullable; lowest g with an error, -1 if none
 * Synchronous error report: unless desc->flags & PREDTOP_NO_SYNC, the call
 * synchronises `cuda_stream` once and returns the status of the lowest bad
 * graph.  With PREDTOP_NO_SYNC it returns PREDTOP_OK after enqueueing, and
 * predtop_dag_status() reports later; graphs with an error get a NaN latency
 * from predtop_stage_forward. */
PREDTOP_API predtop_status predtop_build_dag(const predtop_batch_desc* desc,
                                 const int64_t* node_ptr, const int64_t* edge_ptr,
                                 const int32_t* edge_src, const int32_t* edge_dst,
                                 const predtop_node_feat* feats,
                                 void* workspace, size_t ws_bytes,
                                 int32_t* depth_out, predtop_dag* out,
                                 int32_t* first_bad_graph, void* cuda_stream);

/* Synchronises `cuda_stream` and returns the build status of `dag` (and the
 * lowest bad graph via [host] first_bad_graph, nullable). */
PREDTOP_API predtop_status predtop_dag_status(predtop_dag dag, int32_t* first_bad_graph, void* cuda_stream);

/* Number of uint64 words predtop_reachability writes:
 * sum_g N_g * W_g with W_g = 2 * ceil(N_g / 128).  [host] result. */
PREDTOP_API predtop_status predtop_dag_reach_words(predtop_dag dag, int64_t* words, void* cuda_stream);

/* Copy the closure R to bits_out (device, uint64).  Layout: graph g starts at
 * word offset sum_{h<g} N_h * W_h; row v (caller order) of graph g is W_g
 * words; bit (u % 64) of word (u / 64) of row v is 1 iff v ~> u by >= 1 edge.
 * Padding bits (u >= N_g) are 0.  Rows are 16-byte aligned. */
PREDTOP_API predtop_status predtop_reachability(predtop_dag dag, uint64_t* bits_out, void* cuda_stream);

/* Same layout, for the attention mask M = R | R^T | I (debug / tests). */
PREDTOP_API predtop_status predtop_debug_mask(predtop_dag dag, uint64_t* bits_out, void* cuda_stream);

/* Per-graph block structure of M (debug / tests):
 *  tile_class_out: graph g starts at offset sum_{h<g} T_h^2, T_h = ceil(N_h/128);
 *    entry (qt * T_g + kt) for the 128x128 tile of rows [128qt,..) x cols [128kt,..)
 *    (clipped to N_g): 0 = no allowed pair, 2 = every pair allowed, 1 = otherwise.
 *  pairs_out[G]: |A_g| = popcount(M_g) = N_g + 2 |R_g|.   Both device, nullable. */
PREDTOP_API predtop_status predtop_debug_tiles(predtop_dag dag, uint8_t* tile_class_out,
                                   int64_t* pairs_out, void* cuda_stream);

PREDTOP_API void predtop_dag_destroy(predtop_dag dag);

/* ---------------------------------------------------------------------------
 * DAG-Transformer latency model (SIV-B5).  One model per mesh /
 * parallel configuration.  Readings of unstated details (layer form,
 * PE, head depth, LN eps) are listed in DESIGN.md; summary:
 *   x0 = W_in f(v) + b_in + PE(depth(v))        sinusoidal PE, base 10000
 *   per layer (post-LN encoder layer, ReLU FFN):
 *     a  = concat_h softmax(Q_h K_h^T / sqrt(d_h) + M) V_h ;  (Eqn 1)
 *     h  = LN1(x + W_o a + b_o)
 *     x' = LN2(h + W_2 ReLU(W_1 h + b_1) + b_2)
 *   g  = sum_n x_n   (Eqn 2; mean if pool = 1)
 *   y  = w_o . ReLU(H_2 ReLU(H_1 g + c_1) + c_2) + c_o
 * ------------------------------------------------------------------------- */
enum { PREDTOP_POOL_SUM = 0, PREDTOP_POOL_MEAN = 1 };

typedef struct {
  int32_t num_layers; /* L_m >= 1 (paper: 4) */
  int32_t d_model;    /* d: 32, 64, 128 or 256 (paper: 64) */
  int32_t num_heads;  /* H: d / H must be 16 or 32 */
  int32_t d_ff;       /* FFN width: multiple of 64, <= 1024 */
  int32_t pool;       /* PREDTOP_POOL_SUM (Eqn 2, default) or PREDTOP_POOL_MEAN */
  float ln_eps;       /* LayerNorm epsilon (1e-5) */
} predtop_model_config;

/* Host weight blob: little-endian fp32, concatenated in this order
 * (Linear weights are [out][in], i.e. y = W x + b):
 *   W_in [d][F]  b_in [d]                      F = PREDTOP_NUM_FEATURES
 *   for each layer l = 0..L-1:
 *     W_qkv [3d][d]  b_qkv [3d]   (rows 0..d-1 = Q, d..2d-1 = K, 2d..3d-1 = V;
 *                                  head h owns rows h*d_h .. (h+1)*d_h-1 of each)
 *     W_o [d][d]  b_o [d]
 *     ln1_gamma [d]  ln1_beta [d]
 *     W_1 [d_ff][d]  b_1 [d_ff]
 *     W_2 [d][d_ff]  b_2 [d]
 *     ln2_gamma [d]  ln2_beta [d]
 *   H_1 [d][d] c_1 [d]  H_2 [d][d] c_2 [d]  w_o [d]  c_o [1]
 * The per-layer GEMM weights (W_qkv, W_o, W_1, W_2) are stored on the device
 * as fp16; values that are not fp16-representable are rounded to nearest. */
PREDTOP_API size_t predtop_model_weight_floats(const predtop_model_config* cfg); /* blob length in floats */
PREDTOP_API size_t predtop_model_device_bytes(const predtop_model_config* cfg);  /* device weight bytes */

/* Validates cfg, converts and uploads the blob into caller-allocated device
 * memory (>= predtop_model_device_bytes, 256-byte aligned).  Synchronous. */
PREDTOP_API predtop_status predtop_model_create(const predtop_model_config* cfg,
                                    const float* weights_host, size_t num_floats,
                                    void* device_weights, size_t device_bytes,
                                    predtop_model* out);
PREDTOP_API void predtop_model_destroy(predtop_model model);

/* Device workspace bytes for predtop_stage_forward(model, dag). */
PREDTOP_API size_t predtop_stage_forward_workspace(predtop_model model, predtop_dag dag);

/* latency_out[G] (device, fp32): predicted stage latency of every graph.
 * Deterministic: each graph's value is bit-identical whatever the batch
 * composition, order or size (no split-K, no float atomics). */
PREDTOP_API predtop_status predtop_stage_forward(predtop_model model, predtop_dag dag,
                                     void* workspace, size_t ws_bytes,
                                     float* latency_out, void* cuda_stream);

/* Debug taps for tests: node embeddings after layer `layer` (-1 = x0 after
 * embedding + PE), fp32 [N_tot][d] device.  Valid after predtop_stage_forward
 * ran with the same workspace only for layer = L-1 (the final x); other layers
 * are recomputed by this call. */
PREDTOP_API predtop_status predtop_debug_node_embeddings(predtop_model model, predtop_dag dag,
                                             void* workspace, size_t ws_bytes, int32_t layer,
                                             float* x_out, void* cuda_stream);

/* ---------------------------------------------------------------------------
 * White-box pipeline model, Eqn 4 (SV):
 *   T_p = sum_{i<S_p} t_{p,i} + (B_p - 1) * max_i t_{p,i}
 * plan p uses stages plan_stage[plan_ptr[p] .. plan_ptr[p+1]) (indices into
 * stage_latency), B_p = microbatches[p] microbatches.  Arithmetic is fp64 in a
 * canonical order so T depends only on the multiset of stage latencies:
 * sort the S_p fp32 latencies ascending, sum them in fp64 left to right with
 * round-to-nearest, m = max, T = sum + (double)(B_p-1) * m (two roundings, no
 * FMA).  Invalid plan (S_p < 1, S_p > PREDTOP_MAX_PLAN_STAGES, B_p < 1, a stage
 * index outside [0, num_stages)) -> T_p = NaN and a status word.
 *  plan_ptr[P+1] int64, plan_stage[] int32, microbatches[P] int32,
 *  stage_latency[num_stages] fp32, T_out[P] fp64: all device.
 *  workspace: device, >= predtop_plan_latency_workspace() bytes.
 *  flags: PREDTOP_NO_SYNC or 0 (sync mode returns INVALID_ARG for a bad plan,
 *  and the lowest bad plan index via [host] first_bad_plan, nullable). */
#define PREDTOP_MAX_PLAN_STAGES 64
PREDTOP_API size_t predtop_plan_latency_workspace(void);
PREDTOP_API predtop_status predtop_plan_latency(int64_t num_plans, const int64_t* plan_ptr,
                                    const int32_t* plan_stage, const int32_t* microbatches,
                                    const float* stage_latency, int64_t num_stages,
                                    double* T_out, void* workspace, size_t ws_bytes,
                                    uint32_t flags, int64_t* first_bad_plan,
                                    void* cuda_stream);

/* best_out[1] (device int64) = argmin_p T[p] with ties to the lower index
 * (ranking by (T, plan id), R13).  NaN entries are never chosen unless all
 * are NaN (then -1).  workspace >= predtop_plan_argmin_workspace(n). */
PREDTOP_API size_t predtop_plan_argmin_workspace(int64_t num_plans);
PREDTOP_API predtop_status predtop_plan_argmin(int64_t num_plans, const double* T, int64_t* best_out,
                                   void* workspace, size_t ws_bytes, void* cuda_stream);

/* Misc. */
/* ---------------------------------------------------------------------------
 * Graph pruning (SIV-B4 "Graph Pruning"): "There
 * are several operations whose effects can be stored in the graph even after
 * removing them ... such as reshape and convert_element_type ... We remove
 * these redundant operators from our graphs".  Reading R21: an
 * OPERATOR node (kind 2) whose op id is in pruned_ops is removed; every other
 * node is kept, renumbered in its original order with its record unchanged;
 * kept u gets an edge to kept w iff the raw graph has a path u -> ... -> w of
 * >= 1 edge whose interior nodes are all removed (the removed node's inputs
 * are spliced to its consumers).  Output edges are unique and sorted by
 * (src, dst) within each graph; the output is a batch in the input layout,
 * ready for predtop_build_dag.  Raw primitives outside the Table I vocabulary
 * use op ids >= PREDTOP_NUM_OPS (e.g. the two named by the paper below).
 *  desc, node_ptr, edge_ptr, edge_src, edge_dst, feats: the RAW batch, as for
 *                      predtop_build_dag (device)
 *  pruned_ops[n]       [host] op ids to remove, 1 <= n <= PREDTOP_PRUNE_MAX_OPS
 *  workspace           device, >= predtop_prune_workspace(desc), 256-B aligned
 *  out_node_ptr[G+1], out_edge_ptr[G+1]  device int64
 *  out_src/out_dst     device int32 [edge_capacity], graph-local new ids
 *  out_feats           device [desc->total_nodes] (kept records)
 *  totals              [host] int64[2], nullable: kept nodes, output edges
 *  first_bad_graph     [host] nullable
 * Synchronises `cuda_stream` once (the output sizes).  A raw graph that
 * fails validation (RANGE / SELF_LOOP / CYCLE, TOO_LARGE) -> that status,
 * nothing emitted.  More output edges than edge_capacity -> WORKSPACE (totals
 * still set; call again with a larger buffer).  A graph whose nodes are all
 * removed becomes an empty graph (0 nodes), which predtop_build_dag rejects. */
#define PREDTOP_OP_RESHAPE 64
#define PREDTOP_OP_CONVERT_ELEMENT_TYPE 65
#define PREDTOP_PRUNE_MAX_OPS 16
PREDTOP_API size_t predtop_prune_workspace(const predtop_batch_desc* desc);
PREDTOP_API predtop_status predtop_prune_graphs(const predtop_batch_desc* desc, const int64_t* node_ptr,
                                                const int64_t* edge_ptr, const int32_t* edge_src,
                                                const int32_t* edge_dst, const predtop_node_feat* feats,
                                                const uint16_t* pruned_ops, int32_t num_pruned_ops,
                                                void* workspace, size_t ws_bytes, int64_t* out_node_ptr,
                                                int64_t* out_edge_ptr, int32_t* out_src, int32_t* out_dst,
                                                int64_t edge_capacity, predtop_node_feat* out_feats,
                                                int64_t* totals, int32_t* first_bad_graph, void* cuda_stream);

/* ---------------------------------------------------------------------------
 * Inter-stage plan search over a shared stage table.
 * Alpa's inter-operator optimizer picks the pipeline plan under the
 * 1F1B model; it enumerates all stages on all submeshes; P:222:
 * PredTOP predicts every stage's latency on every mesh, then applies the
 * pipeline model (Eqn 4).  A plan slices layers 0..L-1 into S >= 1
 * contiguous stages [a_s, b_s], gives stage s a choice c_s (a mesh and
 * intra-op configuration, Tables II-III) that uses
 * choice_devices[c_s] devices, uses every device (sum = num_devices), and
 * costs T = sum_s t_s + (B-1) max_s t_s with t_s = table[a_s][b_s][c_s].
 * The call returns, per problem, the minimum T over all plans and one plan
 * attaining it (reading R20 in DESIGN.md; Alpa's t_max-enumeration DP).
 *  num_problems P >= 1; num_layers L in [1, 64]; num_choices K in [1, 32];
 *  choice_devices[K]   [host] int32, each >= 1
 *  num_devices D       [1, 64]
 *  stage_latency       device fp32 [num_tables][K][table_stride]: the latency
 *                      of layers i..j (i <= j) on choice c is element
 *                      tri(i, j) = i*L - i*(i-1)/2 + (j - i) of row c (the
 *                      packed upper triangle, so a stage_forward over the
 *                      L(L+1)/2 stage DAGs in that order writes row c
 *                      directly); an entry is feasible iff finite and >= 0
 *                      (use +inf for a stage that does not fit a mesh)
 *  table_stride        >= L(L+1)/2 (lets row c be an all-gather output)
 *  problem_table[P]    device int32, nullable (then problem p uses table p)
 *  microbatches[P]     device int32, B >= 1
 *  T_out[P]            device fp64: T*; +inf if no plan exists; NaN for an
 *                      invalid problem (table index out of range or B < 1)
 *  num_stages_out[P]   device int32: S of the returned plan (0 if none)
 *  stage_end_out[P][L], stage_choice_out[P][L]  device int32: b_s and c_s for
 *                      s < S (a_0 = 0, a_{s+1} = b_s + 1); the rest untouched
 *  workspace           device, >= predtop_plan_search_workspace(P, L, K) bytes,
 *                      256-byte aligned
 * Exactness: T* is the exact minimum of Eqn 4 over all plans whenever the
 * fp64 sums of fp32 latencies are exact (every feasible latency within a
 * factor 2^24 of the largest), e.g. bit-identical to exhaustive enumeration;
 * among plans with equal T the one returned is the first in (t_max, j, c)
 * order (deterministic).  Host-checkable argument errors -> INVALID_ARG;
 * otherwise stream-ordered, no synchronisation. */
#define PREDTOP_SEARCH_MAX_LAYERS 64
#define PREDTOP_SEARCH_MAX_CHOICES 32
#define PREDTOP_SEARCH_MAX_DEVICES 64
PREDTOP_API size_t predtop_plan_search_workspace(int64_t num_problems, int32_t num_layers, int32_t num_choices);
PREDTOP_API predtop_status predtop_plan_search(int64_t num_problems, int32_t num_layers, int32_t num_choices,
                                               const int32_t* choice_devices, int32_t num_devices,
                                               const float* stage_latency, int64_t table_stride,
                                               int64_t num_tables,
                                               const int32_t* problem_table, const int32_t* microbatches,
                                               double* T_out, int32_t* num_stages_out,
                                               int32_t* stage_end_out, int32_t* stage_choice_out,
                                               void* workspace, size_t ws_bytes, void* cuda_stream);

/* ---------------------------------------------------------------------------
 * Training (SIV-B6-8; the training phase of P:219)
 * of one DAG-Transformer on (stage DAG, latency) pairs:
 *   loss  L = (1/G) sum_g |y_hat_g - y_g|              MAE, Eqn 3
 *   Adam (beta1 0.9, beta2 0.999, eps 1e-8)    predtop_train_adam
 *   cosine learning-rate decay 1e-3 -> 0 and early stopping (patience 200,
 *   P:186) are host logic of the caller (paper_conf_ipps_acharyas25_b200/train.py).
 * The training path computes in fp32 throughout (forward with every
 * activation kept, backward, optimizer): fp32 master weights, no fp16
 * rounding; dense GEMMs through cuBLAS (plain library GEMMs), the masked
 * attention forward/backward, LayerNorm, pooling/head and loss in this
 * library's kernels.  Deterministic (no float atomics).
 *
 * The state holds four fp32 copies of the weight blob (same order and length
 * as predtop_model_weight_floats): parameters, gradient, Adam m and v, in
 * caller-allocated device memory of predtop_train_state_bytes (256-byte
 * aligned).  Limits: d_model <= 256, d_model / num_heads <= 32, d_ff <= 4096.
 * ------------------------------------------------------------------------- */
typedef struct predtop_train_s* predtop_train;

PREDTOP_API size_t predtop_train_state_bytes(const predtop_model_config* cfg);
/* Uploads weights_host (num_floats = predtop_model_weight_floats) as the fp32
 * parameters, zeroes gradient and moments.  Synchronous. */
PREDTOP_API predtop_status predtop_train_create(const predtop_model_config* cfg, const float* weights_host,
                                                size_t num_floats, void* device_state, size_t state_bytes,
                                                predtop_train* out);
PREDTOP_API void predtop_train_destroy(predtop_train tr);
/* Device workspace bytes for predtop_train_grad on this batch. */
PREDTOP_API size_t predtop_train_workspace(predtop_train tr, predtop_dag dag);
/* Forward (fp32, activations kept), MAE loss against y_true[G] (device fp32)
 * and backward into the state's gradient (overwritten: the gradient of the
 * batch mean).  loss_out[1], y_pred_out[G] (device fp32) nullable.  Every
 * graph of the batch must have status OK (build the DAG with the default
 * synchronous validation); otherwise PREDTOP_ERR_INVALID_ARG. */
PREDTOP_API predtop_status predtop_train_grad(predtop_train tr, predtop_dag dag, const float* y_true,
                                              void* workspace, size_t ws_bytes, float* loss_out,
                                              float* y_pred_out, void* cuda_stream);
/* One Adam update of the parameters from the state's gradient (step >= 1 is
 * the bias-correction count), torch.optim.Adam semantics (no weight decay):
 *   m = b1 m + (1-b1) g,  v = b2 v + (1-b2) g^2,
 *   p -= lr / (1 - b1^step) * m / (sqrt(v) / sqrt(1 - b2^step) + eps). */
PREDTOP_API predtop_status predtop_train_adam(predtop_train tr, float lr, int32_t step, float beta1,
                                              float beta2, float eps, void* cuda_stream);
/* Device pointers of the state's fp32 blobs (which: 0 parameters, 1
 * gradient, 2 m, 3 v), e.g. to copy the trained weights out or to compare the
 * gradient.  NULL for a bad handle or index. */
PREDTOP_API float* predtop_train_buffer(predtop_train tr, int32_t which);

PREDTOP_API const char* predtop_status_string(predtop_status s);
PREDTOP_API const char* predtop_last_error(void); /* thread-local */
PREDTOP_API int predtop_abi_version(void);
/* Number of kernels this library has launched in this process (all entry
 * points).  Lets callers count launches inside a timed region. */
PREDTOP_API int64_t predtop_launch_count(void);

/* Optional per-kernel timing.  When enabled, every launch site records a CUDA
 * event pair on its launching stream.  predtop_profile_read synchronises on
 * the recorded events, writes the accumulated milliseconds and launch counts
 * per kernel kind (ms[k], launches[k], k < min(max_kinds, kinds)), resets the
 * accumulators and returns the number of kinds; predtop_profile_kind_name(k)
 * names kind k.  [host] arrays, nullable. */
PREDTOP_API void predtop_profile_enable(int on);
PREDTOP_API int predtop_profile_read(double* ms, int64_t* launches, int max_kinds);
PREDTOP_API const char* predtop_profile_kind_name(int kind);

#ifdef __cplusplus
}
#endif
#endif /* PREDTOP_H */
