/*
 * oracle.h -- plain CPU fp64 oracle of the PredTOP prediction path.
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing in the product path (the CUDA library
 * and its Python binding) may include, link, import or call this code; only
 * tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference leg use it.  It shares no code, header, table or constant
 * generator with the CUDA path; both read the same documented input formats
 * (include/predtop.h: node record, packed graphs, weight blob order), which
 * this file re-declares independently.
 *
 * Every function cites the passage of the paper (PAPER.md line "P:n") it
 * follows.  Readings of passages the paper leaves open are the ones listed in
 * DESIGN.md ("Readings") and are named R1..R16 below.
 *
 * Parity pins (tests/test_oracle_*.py): brute force on all small DAGs, closed
 * forms, torch float64 library special cases (nn.TransformerEncoderLayer,
 * scaled_dot_product_attention), invariances, the hand-worked Fig. 6 example.
 */
#ifndef PREDTOP_ORACLE_H
#define PREDTOP_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Table I record; layout fixed by the ABI: 20 bytes. */
typedef struct {
  uint16_t op;
  uint8_t dtype;
  uint8_t kind;
  uint32_t dims[4];
} orc_feat;

#define ORC_NUM_OPS 64
#define ORC_NUM_DIMS 4
#define ORC_NUM_DTYPES 8
#define ORC_NUM_KINDS 4
#define ORC_F (ORC_NUM_OPS + ORC_NUM_DIMS + ORC_NUM_DTYPES + ORC_NUM_KINDS)

typedef struct {
  int L;        /* DAG-Transformer layers */
  int d;        /* embedding dimension */
  int H;        /* heads (R8) */
  int d_ff;     /* FFN width (R6) */
  int pool;     /* 0 = global add pool (Eqn 2), 1 = mean (R11 flag) */
  double ln_eps;
} orc_cfg;

/* status codes (same values as the ABI's, re-declared) */
#define ORC_OK 0
#define ORC_RANGE (-2)
#define ORC_SELF_LOOP (-3)
#define ORC_CYCLE (-4)

int orc_validate(int n, int e, const int32_t* src, const int32_t* dst);
void orc_depth(int n, int e, const int32_t* src, const int32_t* dst, int32_t* depth);
int orc_row_words(int n);
void orc_reach(int n, int e, const int32_t* src, const int32_t* dst, uint64_t* R);
void orc_reach_k(int n, int e, const int32_t* src, const int32_t* dst, int k, uint64_t* R);
void orc_mask(int n, const uint64_t* R, uint64_t* M);
int64_t orc_tiles(int n, const uint64_t* M, uint8_t* cls);

long orc_blob_floats(const orc_cfg* c);
void orc_features(int n, const orc_feat* feats, double* f);
void orc_embed(const orc_cfg* c, const float* blob, int n, const orc_feat* feats,
               const int32_t* depth, double* x0);
void orc_attention(const orc_cfg* c, const float* blob, int layer, int n, const uint64_t* M,
                   const double* x, double* concat_out);
void orc_layer(const orc_cfg* c, const float* blob, int layer, int n, const uint64_t* M,
               const double* x_in, double* x_out);
/* The same layer split into row-wise pieces (orc_layer is their composition), */
/* so one large graph can be evaluated row block by row block (16k config).    */
void orc_qkv_rows(const orc_cfg* c, const float* blob, int layer, int r0, int r1, const double* x,
                  double* qkv);
void orc_attention_rows(const orc_cfg* c, int n, const uint64_t* M, const double* qkv, int r0, int r1,
                        double* concat_out);
void orc_layer_post_rows(const orc_cfg* c, const float* blob, int layer, int r0, int r1, const double* a,
                         const double* x_in, double* x_out);
double orc_readout(const orc_cfg* c, const float* blob, int n, const double* x);
int orc_forward(const orc_cfg* c, const float* blob, int n, int e, const int32_t* src,
                const int32_t* dst, const orc_feat* feats, double* y, double* taps);
int orc_forward_k(const orc_cfg* c, const float* blob, int n, int e, const int32_t* src,
                  const int32_t* dst, const orc_feat* feats, int k, double* y, double* taps);

/* Training: y of one graph and grad += dy * dy/dtheta */
/* over the whole weight blob (same float order), fp64.                            */
int orc_grad(const orc_cfg* c, const float* blob, int n, int e, const int32_t* src, const int32_t* dst,
             const orc_feat* feats, double dy, double* y, double* grad);

void orc_plan_T(int64_t P, const int64_t* plan_ptr, const int32_t* plan_stage,
                const int32_t* B, const float* t, int64_t num_stages, double* T);
int64_t orc_argmin(int64_t n, const double* T);
int orc_prune(int n, int e, const int32_t* src, const int32_t* dst, const orc_feat* feats,
              const uint16_t* ops, int n_ops, int32_t* nk_out, int32_t* out_src, int32_t* out_dst,
              int64_t* ne_out, orc_feat* out_feats);
double orc_plan_search(int L, int K, const int32_t* dev, int D, const float* t, int B,
                       int32_t* S_out, int32_t* stage_end, int32_t* stage_choice);

#ifdef __cplusplus
}
#endif
#endif
