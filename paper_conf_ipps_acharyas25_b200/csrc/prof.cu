// prof.cu -- optional per-kernel CUDA-event timing of every launch site
// (predtop_profile_enable / predtop_profile_read).  Used by bench.py to time
// the dominant kernel live, on the stream it is launched on.
#include <mutex>
#include <vector>

#include "internal.h"

namespace predtop {

namespace {
struct Rec {
  int kind;
  cudaEvent_t a, b;
};
std::mutex g_mu;
bool g_on = false;
std::vector<Rec> g_recs;
std::vector<cudaEvent_t> g_pool;
double g_ms[PK_COUNT];
int64_t g_cnt[PK_COUNT];

cudaEvent_t take_event() {
  if (!g_pool.empty()) {
    cudaEvent_t e = g_pool.back();
    g_pool.pop_back();
    return e;
  }
  cudaEvent_t e = nullptr;
  cudaEventCreate(&e);
  return e;
}

const char* kNames[PK_COUNT] = {
    "dag_meta", "dag_depth", "dag_closure", "dag_mask", "dag_classify", "dag_work",
    "pe_table", "embed", "gemm_qkv", "attention", "gemm_oproj_ln", "gemm_ffn1",
    "gemm_ffn2_ln", "readout", "plan_latency", "plan_argmin", "copy", "layer_tail", "dag_small", "dag_flags",
    "search_cand", "search_pick", "prune"};
}  // namespace

ProfScope::ProfScope(int k, cudaStream_t s) : kind(k), st(s) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (!g_on) return;
  cudaEvent_t e = take_event();
  if (e && cudaEventRecord(e, s) == cudaSuccess) ev0 = e;
}

ProfScope::~ProfScope() {
  if (!ev0) return;
  std::lock_guard<std::mutex> lk(g_mu);
  cudaEvent_t e = take_event();
  if (e && cudaEventRecord(e, st) == cudaSuccess) g_recs.push_back({kind, (cudaEvent_t)ev0, e});
}

}  // namespace predtop

using namespace predtop;

extern "C" {

void predtop_profile_enable(int on) {
  std::lock_guard<std::mutex> lk(g_mu);
  g_on = on != 0;
}

int predtop_profile_read(double* ms, int64_t* launches, int max_kinds) {
  std::lock_guard<std::mutex> lk(g_mu);
  for (Rec& r : g_recs) {
    float t = 0.f;
    if (cudaEventSynchronize(r.b) == cudaSuccess && cudaEventElapsedTime(&t, r.a, r.b) == cudaSuccess) {
      g_ms[r.kind] += t;
      g_cnt[r.kind] += 1;
    }
    g_pool.push_back(r.a);
    g_pool.push_back(r.b);
  }
  g_recs.clear();
  cudaGetLastError();
  const int n = max_kinds < PK_COUNT ? max_kinds : PK_COUNT;
  for (int k = 0; k < n; ++k) {
    if (ms) ms[k] = g_ms[k];
    if (launches) launches[k] = g_cnt[k];
  }
  for (int k = 0; k < PK_COUNT; ++k) {
    g_ms[k] = 0.0;
    g_cnt[k] = 0;
  }
  return PK_COUNT;
}

const char* predtop_profile_kind_name(int kind) {
  return (kind >= 0 && kind < PK_COUNT) ? kNames[kind] : "";
}

}  // extern "C"
