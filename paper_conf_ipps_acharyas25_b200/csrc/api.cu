// api.cu -- the extern "C" boundary of libpredtop (include/predtop.h):
// argument validation, workspace carving, handle management and the launch
// sequence of each entry point.  All arithmetic of the method runs in the
// kernels of dag.cu, embed_readout.cu, gemm.cu, attention.cu and plan.cu.
#include <atomic>
#include <climits>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <new>
#include <utility>
#include <vector>

#include "internal.h"

namespace predtop {

static thread_local char g_err[1024] = "";
static std::atomic<int64_t> g_launches{0};

void note_launch(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

void set_error(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
}

cudaError_t smem_attr(const void* func, int bytes) {
  if (bytes <= 48 * 1024) return cudaSuccess;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  static std::mutex mu;
  static std::map<std::pair<int, const void*>, int> done;
  std::lock_guard<std::mutex> lock(mu);
  int& have = done[{dev, func}];
  if (have >= bytes) return cudaSuccess;
  e = cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  if (e == cudaSuccess) have = bytes;
  return e;
}

int num_sms() {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return 0;
  static std::atomic<int> cache[64] = {};
  if (dev >= 0 && dev < 64 && cache[dev].load()) return cache[dev].load();
  int n = 0;
  if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return 0;
  if (dev >= 0 && dev < 64) cache[dev] = n;
  return n;
}

static inline cudaStream_t S(void* s) { return reinterpret_cast<cudaStream_t>(s); }

// ------------------------------------------------------------ DAG workspace
struct DagBounds {
  int64_t words, tiles, qtiles, bflags;
  int32_t max_words;
};

static bool dag_bounds(const predtop_batch_desc* b, DagBounds* o) {
  if (!b || b->num_graphs < 1 || b->total_nodes < b->num_graphs || b->total_edges < 0 ||
      b->max_nodes < 1)
    return false;
  const int64_t maxn = std::min<int64_t>(b->max_nodes, PREDTOP_MAX_NODES);
  const int64_t T = ceil_div(maxn, 128);
  o->max_words = (int32_t)(2 * T);
  o->words = b->total_nodes * 2 * T;
  o->qtiles = ceil_div(b->total_nodes, 128) + b->num_graphs;
  o->tiles = o->qtiles * T;
  o->bflags = (ceil_div(b->total_nodes, 16) + b->num_graphs) * ceil_div(maxn, 64);
  return true;
}

static size_t carve_dag(const predtop_batch_desc* b, const DagBounds& bd, void* ws, bool own_depth,
                        DagDev* d) {
  Carver c(ws);
  const int64_t G = b->num_graphs, N = b->total_nodes, E = std::max<int64_t>(b->total_edges, 1);
  DagDev t{};
  t.status = c.take<int32_t>(G);
  t.num_levels = c.take<int32_t>(G);
  t.row_off = c.take<int64_t>(G + 1);
  t.tile_off = c.take<int64_t>(G + 1);
  t.qtile_off = c.take<int32_t>(G + 1);
  t.pairs = c.take<int64_t>(G);
  t.first_bad = c.take<int32_t>(1);
  t.depth = own_depth ? c.take<int32_t>(N) : nullptr;
  t.topo = c.take<int32_t>(N);
  t.level_ptr = c.take<int32_t>(N + G);
  t.succ_off = c.take<int32_t>(N + G);
  t.succ = c.take<int32_t>(E);
  t.indeg = c.take<int32_t>(N);
  t.rec = c.take<int4>(N);
  t.R = c.take<uint64_t>(bd.words);
  t.M = c.take<uint64_t>(bd.words);
  t.tile_cnt = c.take<int32_t>(bd.tiles);
  t.tile_cls = c.take<uint8_t>(bd.tiles);
  t.work = c.take<int2>(bd.qtiles);
  t.bflag_off = c.take<int64_t>(G + 1);
  t.bflag = c.take<uint8_t>(bd.bflags);
  if (d) *d = t;
  return align_up(c.used, 256);
}

// ------------------------------------------------------------ forward workspace
struct FwdWs {
  float* x32;
  __half* x16;
  __half* qkv;
  __half* att;
  __half* hid;
  float* pe;
};

static size_t carve_fwd(const predtop_model_s* m, const predtop_dag_s* dag, void* ws, FwdWs* o) {
  Carver c(ws);
  const int64_t N = dag->desc.total_nodes;
  const int d = m->cfg.d_model, f = m->cfg.d_ff;
  FwdWs w{};
  w.x32 = c.take<float>((size_t)N * d, 1024);
  w.x16 = c.take<__half>((size_t)N * d, 1024);
  w.qkv = c.take<__half>((size_t)N * 3 * d, 1024);
  w.att = c.take<__half>((size_t)N * d, 1024);
  w.hid = c.take<__half>((size_t)N * f, 1024);
  w.pe = c.take<float>((size_t)std::min<int64_t>(dag->desc.max_nodes, PREDTOP_MAX_NODES) * d, 1024);
  if (o) *o = w;
  return align_up(c.used, 256);
}

// ------------------------------------------------------------ model layout
static int kch_for(int K) { return K % 64 == 0 ? 64 : 32; }

static bool model_cfg_ok(const predtop_model_config* c) {
  if (!c) return false;
  if (c->num_layers < 1 || c->num_layers > kMaxLayers) return false;
  if (!(c->d_model == 32 || c->d_model == 64 || c->d_model == 128 || c->d_model == 256)) return false;
  if (c->num_heads < 1 || c->d_model % c->num_heads) return false;
  const int dh = c->d_model / c->num_heads;
  if (dh != 16 && dh != 32) return false;
  if (c->d_ff < 64 || c->d_ff > 1024 || c->d_ff % 64) return false;
  if (c->pool != PREDTOP_POOL_SUM && c->pool != PREDTOP_POOL_MEAN) return false;
  if (!(c->ln_eps > 0.f)) return false;
  if (gemm_pick_bn(3 * c->d_model) == 0 || gemm_pick_bn(c->d_ff) == 0) return false;
  return true;
}

static size_t blob_floats(const predtop_model_config* c) {
  const size_t d = c->d_model, f = c->d_ff, F = PREDTOP_NUM_FEATURES;
  const size_t layer = 3 * d * d + 3 * d + d * d + d + 2 * d + f * d + f + d * f + d + 2 * d;
  return d * F + d + (size_t)c->num_layers * layer + 2 * (d * d + d) + d + 1;
}

static size_t carve_model(const predtop_model_config* c, void* base, predtop_model_s* m) {
  Carver k(base);
  const size_t d = c->d_model, f = c->d_ff, F = PREDTOP_NUM_FEATURES;
  predtop_model_s t{};
  t.W_inT = k.take<float>(F * d);
  t.b_in = k.take<float>(d);
  for (int l = 0; l < c->num_layers; ++l) {
      LayerDev& L = t.layer[l];
      L.Wqkv = k.take<__half>(3 * d * d, 1024);
      L.bqkv = k.take<float>(3 * d);
      L.Wo = k.take<__half>(d * d, 1024);
      L.bo = k.take<float>(d);
      L.g1 = k.take<float>(d);
      L.be1 = k.take<float>(d);
      L.W1 = k.take<__half>(f * d, 1024);
      L.b1 = k.take<float>(f);
      L.W2 = k.take<__half>(d * f, 1024);
      L.b2 = k.take<float>(d);
      L.g2 = k.take<float>(d);
      L.be2 = k.take<float>(d);
  }
  t.H1T = k.take<float>(d * d);
  t.c1 = k.take<float>(d);
  t.H2T = k.take<float>(d * d);
  t.c2 = k.take<float>(d);
  t.w_o = k.take<float>(d);
  t.c_o = k.take<float>(1);
  if (m) {
    t.cfg = *c;
    *m = t;
  }
  return align_up(k.used, 256);
}

static bool device_ok() {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) {
    set_error("no CUDA device");
    return false;
  }
  // cached per device: cudaGetDeviceProperties costs milliseconds of host
  // time, and this runs on every build (the eager sweep builds ~100 chunks)
  static std::atomic<int> ok_dev[64] = {};  // 0 unknown, 1 ok, -1 not sm_100
  if (dev >= 0 && dev < 64 && ok_dev[dev].load() == 1) return true;
  // only sm_100a SASS is built: compute capability exactly 10.0 (sm_103 / sm_12x would fail at launch)
  int major = 0, minor = 0;
  if (cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev) != cudaSuccess ||
      cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev) != cudaSuccess || major != 10 ||
      minor != 0) {
    set_error("libpredtop is built for sm_100a only and needs a compute capability 10.0 (B200) device");
    cudaGetLastError();
    if (dev >= 0 && dev < 64) ok_dev[dev] = -1;
    return false;
  }
  if (dev >= 0 && dev < 64) ok_dev[dev] = 1;
  return true;
}

}  // namespace predtop

using namespace predtop;

extern "C" {

int predtop_abi_version(void) { return PREDTOP_ABI_VERSION; }
int64_t predtop_launch_count(void) { return g_launches.load(); }
const char* predtop_last_error(void) { return g_err; }

const char* predtop_status_string(predtop_status s) {
  switch (s) {
    case PREDTOP_OK: return "ok";
    case PREDTOP_ERR_INVALID_ARG: return "invalid argument";
    case PREDTOP_ERR_RANGE: return "edge endpoint out of range";
    case PREDTOP_ERR_SELF_LOOP: return "self loop";
    case PREDTOP_ERR_CYCLE: return "graph has a cycle";
    case PREDTOP_ERR_TOO_LARGE: return "graph too large";
    case PREDTOP_ERR_WORKSPACE: return "workspace too small";
    case PREDTOP_ERR_CUDA: return "CUDA error";
    case PREDTOP_ERR_UNSUPPORTED: return "unsupported configuration";
  }
  return "unknown status";
}

size_t predtop_build_dag_workspace(const predtop_batch_desc* desc) {
  DagBounds bd;
  if (!dag_bounds(desc, &bd)) return 0;
  return carve_dag(desc, bd, nullptr, true, nullptr);
}

predtop_status predtop_build_dag(const predtop_batch_desc* desc, const int64_t* node_ptr,
                                 const int64_t* edge_ptr, const int32_t* edge_src,
                                 const int32_t* edge_dst, const predtop_node_feat* feats,
                                 void* workspace, size_t ws_bytes, int32_t* depth_out,
                                 predtop_dag* out, int32_t* first_bad_graph, void* cuda_stream) {
  if (first_bad_graph) *first_bad_graph = -1;
  if (!out) { set_error("out is NULL"); return PREDTOP_ERR_INVALID_ARG; }
  *out = nullptr;
  DagBounds bd;
  if (!dag_bounds(desc, &bd)) { set_error("invalid batch descriptor"); return PREDTOP_ERR_INVALID_ARG; }
  if (desc->hops < 0) { set_error("hops %d < 0", desc->hops); return PREDTOP_ERR_INVALID_ARG; }
  if (desc->max_nodes > PREDTOP_MAX_NODES) {
    set_error("max_nodes %d > PREDTOP_MAX_NODES", desc->max_nodes);
    return PREDTOP_ERR_TOO_LARGE;
  }
  if (!node_ptr || !edge_ptr || !feats || (desc->total_edges > 0 && (!edge_src || !edge_dst)) ||
      !workspace) {
    set_error("NULL array argument");
    return PREDTOP_ERR_INVALID_ARG;
  }
  if (((uintptr_t)workspace & 255) || ws_bytes < predtop_build_dag_workspace(desc)) {
    set_error("workspace too small or not 256-byte aligned (%zu < %zu)", ws_bytes,
              predtop_build_dag_workspace(desc));
    return PREDTOP_ERR_WORKSPACE;
  }
  if (!device_ok()) return PREDTOP_ERR_CUDA;
  predtop_dag_s* dag = new (std::nothrow) predtop_dag_s();
  if (!dag) { set_error("out of host memory"); return PREDTOP_ERR_INVALID_ARG; }
  dag->desc = *desc;
  carve_dag(desc, bd, workspace, depth_out == nullptr, &dag->d);
  dag->d.node_ptr = node_ptr;
  dag->d.edge_ptr = edge_ptr;
  dag->d.src = edge_src;
  dag->d.dst = edge_dst;
  dag->d.feats = feats;
  dag->d.hops = desc->hops;
  if (depth_out) dag->d.depth = depth_out;
  dag->words_bound = bd.words;
  dag->tiles_bound = bd.tiles;
  dag->qtiles_bound = bd.qtiles;
  dag->bflags_bound = bd.bflags;
  dag->max_words = bd.max_words;
  *out = dag;
  predtop_status st = dag_build_launch(dag, S(cuda_stream));
  if (st != PREDTOP_OK) return st;
  if (desc->flags & PREDTOP_NO_SYNC) return PREDTOP_OK;
  return predtop_dag_status(dag, first_bad_graph, cuda_stream);
}

predtop_status predtop_dag_status(predtop_dag dag, int32_t* first_bad_graph, void* cuda_stream) {
  if (first_bad_graph) *first_bad_graph = -1;
  if (!dag) { set_error("dag is NULL"); return PREDTOP_ERR_INVALID_ARG; }
  int32_t fb = INT_MAX;
  PT_CUDA_TRY(cudaMemcpyAsync(&fb, dag->d.first_bad, sizeof(fb), cudaMemcpyDeviceToHost, S(cuda_stream)));
  PT_CUDA_TRY(cudaStreamSynchronize(S(cuda_stream)));
  if (fb == INT_MAX) return PREDTOP_OK;
  int32_t code = 0;
  PT_CUDA_TRY(cudaMemcpy(&code, dag->d.status + fb, sizeof(code), cudaMemcpyDeviceToHost));
  if (first_bad_graph) *first_bad_graph = fb;
  set_error("graph %d: %s", fb, predtop_status_string((predtop_status)code));
  return (predtop_status)code;
}

predtop_status predtop_dag_reach_words(predtop_dag dag, int64_t* words, void* cuda_stream) {
  if (!dag || !words) { set_error("NULL argument"); return PREDTOP_ERR_INVALID_ARG; }
  PT_CUDA_TRY(cudaMemcpyAsync(words, dag->d.row_off + dag->desc.num_graphs, sizeof(int64_t),
                              cudaMemcpyDeviceToHost, S(cuda_stream)));
  PT_CUDA_TRY(cudaStreamSynchronize(S(cuda_stream)));
  return PREDTOP_OK;
}

predtop_status predtop_reachability(predtop_dag dag, uint64_t* bits_out, void* cuda_stream) {
  if (!dag || !bits_out) { set_error("NULL argument"); return PREDTOP_ERR_INVALID_ARG; }
  return dag_copy_bits(dag, dag->d.R, bits_out, S(cuda_stream));
}

predtop_status predtop_debug_mask(predtop_dag dag, uint64_t* bits_out, void* cuda_stream) {
  if (!dag || !bits_out) { set_error("NULL argument"); return PREDTOP_ERR_INVALID_ARG; }
  return dag_copy_bits(dag, dag->d.M, bits_out, S(cuda_stream), /*unperm=*/true);
}

predtop_status predtop_debug_tiles(predtop_dag dag, uint8_t* tile_class_out, int64_t* pairs_out,
                                   void* cuda_stream) {
  if (!dag) { set_error("dag is NULL"); return PREDTOP_ERR_INVALID_ARG; }
  const int G = dag->desc.num_graphs;
  int64_t ntiles = 0;
  PT_CUDA_TRY(cudaMemcpyAsync(&ntiles, dag->d.tile_off + G, sizeof(ntiles), cudaMemcpyDeviceToHost,
                              S(cuda_stream)));
  PT_CUDA_TRY(cudaStreamSynchronize(S(cuda_stream)));
  if (tile_class_out && ntiles)
    PT_CUDA_TRY(cudaMemcpyAsync(tile_class_out, dag->d.tile_cls, (size_t)ntiles,
                                cudaMemcpyDeviceToDevice, S(cuda_stream)));
  if (pairs_out)
    PT_CUDA_TRY(cudaMemcpyAsync(pairs_out, dag->d.pairs, sizeof(int64_t) * G,
                                cudaMemcpyDeviceToDevice, S(cuda_stream)));
  return PREDTOP_OK;
}

void predtop_dag_destroy(predtop_dag dag) { delete dag; }

// ------------------------------------------------------------------- model
size_t predtop_model_weight_floats(const predtop_model_config* cfg) {
  return model_cfg_ok(cfg) ? blob_floats(cfg) : 0;
}

size_t predtop_model_device_bytes(const predtop_model_config* cfg) {
  return model_cfg_ok(cfg) ? carve_model(cfg, nullptr, nullptr) : 0;
}

predtop_status predtop_model_create(const predtop_model_config* cfg, const float* w,
                                    size_t num_floats, void* device_weights,
                                    size_t device_bytes, predtop_model* out) {
  if (!out) { set_error("out is NULL"); return PREDTOP_ERR_INVALID_ARG; }
  *out = nullptr;
  if (!cfg || !model_cfg_ok(cfg)) {
    set_error("unsupported model config (d in {32,64,128,256}, d/H in {16,32}, d_ff %% 64 == 0 <= 1024)");
    return PREDTOP_ERR_UNSUPPORTED;
  }
  if (!w || num_floats != blob_floats(cfg)) {
    set_error("weight blob has %zu floats, expected %zu", num_floats, blob_floats(cfg));
    return PREDTOP_ERR_INVALID_ARG;
  }
  const size_t need = carve_model(cfg, nullptr, nullptr);
  if (!device_weights || device_bytes < need || ((uintptr_t)device_weights & 255)) {
    set_error("device weight buffer too small or misaligned (%zu < %zu)", device_bytes, need);
    return PREDTOP_ERR_WORKSPACE;
  }
  if (!device_ok()) return PREDTOP_ERR_CUDA;
  predtop_model_s* m = new (std::nothrow) predtop_model_s();
  if (!m) { set_error("out of host memory"); return PREDTOP_ERR_INVALID_ARG; }
  carve_model(cfg, device_weights, m);
  // Stage the device image on the host, then one synchronous copy.
  std::vector<unsigned char> img(need, 0);
  char* dev0 = (char*)device_weights;
  auto H = [&](void* devp) { return (void*)(img.data() + ((char*)devp - dev0)); };
  const int d = cfg->d_model, f = cfg->d_ff, F = PREDTOP_NUM_FEATURES;
  const float* p = w;
  auto f32 = [&](float* dst, size_t n) { std::memcpy(H(dst), p, n * 4); p += n; };
  auto f16 = [&](__half* dst, size_t n) {
    __half* h = (__half*)H(dst);
    for (size_t i = 0; i < n; ++i) h[i] = __float2half_rn(p[i]);
    p += n;
  };
  auto f32T = [&](float* dst, int rows, int cols) {  // [rows][cols] -> [cols][rows]
    float* h = (float*)H(dst);
    for (int r = 0; r < rows; ++r)
      for (int c = 0; c < cols; ++c) h[(size_t)c * rows + r] = p[(size_t)r * cols + c];
    p += (size_t)rows * cols;
  };
  f32T(m->W_inT, d, F);
  f32(m->b_in, d);
  for (int l = 0; l < cfg->num_layers; ++l) {
    LayerDev& L = m->layer[l];
    f16(L.Wqkv, (size_t)3 * d * d);
    f32(L.bqkv, 3 * d);
    f16(L.Wo, (size_t)d * d);
    f32(L.bo, d);
    f32(L.g1, d);
    f32(L.be1, d);
    f16(L.W1, (size_t)f * d);
    f32(L.b1, f);
    f16(L.W2, (size_t)d * f);
    f32(L.b2, d);
    f32(L.g2, d);
    f32(L.be2, d);
  }
  f32T(m->H1T, d, d);
  f32(m->c1, d);
  f32T(m->H2T, d, d);
  f32(m->c2, d);
  f32(m->w_o, d);
  f32(m->c_o, 1);
  cudaError_t e = cudaMemcpy(device_weights, img.data(), need, cudaMemcpyHostToDevice);
  if (e != cudaSuccess) {
    set_error("weight upload failed: %s", cudaGetErrorString(e));
    delete m;
    return PREDTOP_ERR_CUDA;
  }
  m->bn_qkv = gemm_pick_bn(3 * d);
  m->bn_ff1 = gemm_pick_bn(f);
  for (int l = 0; l < cfg->num_layers; ++l) {
    LayerDev& L = m->layer[l];
    bool ok = encode_tma_2d_f16(&L.tm_qkv, L.Wqkv, d, 3 * d, kch_for(d), m->bn_qkv) &&
              encode_tma_2d_f16(&L.tm_o, L.Wo, d, d, kch_for(d), d) &&
              encode_tma_2d_f16(&L.tm_1, L.W1, d, f, kch_for(d), m->bn_ff1) &&
              encode_tma_2d_f16(&L.tm_2, L.W2, f, d, kch_for(f), d) &&
              (f < 128 || encode_tma_2d_f16(&L.tm_1c, L.W1, d, f, kch_for(d), 128)) &&
              (f < 64 || encode_tma_2d_f16(&L.tm_1h, L.W1, d, f, kch_for(d), 64)) &&
              (d != 256 || (encode_tma_2d_f16(&L.tm_o32, L.Wo, d, d, 32, d) &&
                            encode_tma_2d_f16(&L.tm_2_32, L.W2, f, d, 32, d)));
    if (!ok) {
      delete m;
      return PREDTOP_ERR_CUDA;
    }
  }
  *out = m;
  return PREDTOP_OK;
}

void predtop_model_destroy(predtop_model model) { delete model; }

size_t predtop_stage_forward_workspace(predtop_model model, predtop_dag dag) {
  if (!model || !dag) return 0;
  return carve_fwd(model, dag, nullptr, nullptr);
}

// The fused layer tail covers d in {64, 128} (layer.cu / layer2.cu) and
// d = 256 (layer256.cu); PREDTOP_UNFUSED=1 forces the three-GEMM path (tests
// compare the two).
static bool use_fused_tail(int d, int dff) {
  const char* e = getenv("PREDTOP_UNFUSED");
  const bool unfused = e && e[0] == '1';
  return !unfused && (layer_tail_supported(d, dff) || layer_tail256_supported(d, dff));
}

// d = 128: the two-CTA-per-SM tail (layer2.cu); PREDTOP_TAIL_V1=1 selects the
// one-CTA kernel of layer.cu instead (tests compare the two).
static bool use_tail_v2(int d, int dff) {
  const char* e = getenv("PREDTOP_TAIL_V1");
  return !(e && e[0] == '1') && layer_tail2_supported(d, dff);
}


static predtop_status forward_impl(predtop_model m, predtop_dag dag, void* ws, size_t ws_bytes,
                                   int last_layer, float* latency_out, float* x_out,
                                   cudaStream_t st) {
  if (!m || !dag || !ws) { set_error("NULL argument"); return PREDTOP_ERR_INVALID_ARG; }
  if (((uintptr_t)ws & 255) || ws_bytes < carve_fwd(m, dag, nullptr, nullptr)) {
    set_error("forward workspace too small or misaligned");
    return PREDTOP_ERR_WORKSPACE;
  }
  FwdWs w;
  carve_fwd(m, dag, ws, &w);
  const int d = m->cfg.d_model, f = m->cfg.d_ff, H = m->cfg.num_heads;
  const int64_t Ntot = dag->desc.total_nodes;
  if (Ntot > INT_MAX) { set_error("too many nodes"); return PREDTOP_ERR_TOO_LARGE; }
  const int M = (int)Ntot;
  CUtensorMap tm_x16, tm_att, tm_hid;
  if (!encode_tma_2d_f16(&tm_x16, w.x16, d, Ntot, kch_for(d), 128) ||
      !encode_tma_2d_f16(&tm_att, w.att, d, Ntot, kch_for(d), 128) ||
      !encode_tma_2d_f16(&tm_hid, w.hid, f, Ntot, kch_for(f), 128))
    return PREDTOP_ERR_CUDA;
  // d = 256 LayerNorm GEMMs: the fp32 residual tile takes 128 KB of staging,
  // so 64-wide K-slices leave a one-stage operand ring; 32-wide slices give 3
  const bool ln32 = d == 256;
  CUtensorMap tm_att32, tm_hid32;
  if (ln32 && (!encode_tma_2d_f16(&tm_att32, w.att, d, Ntot, 32, 128) ||
               !encode_tma_2d_f16(&tm_hid32, w.hid, f, Ntot, 32, 128)))
    return PREDTOP_ERR_CUDA;
  predtop_status s;
  const int pe_rows = std::min<int>(dag->desc.max_nodes, PREDTOP_MAX_NODES);
  if ((s = pe_table_launch(w.pe, pe_rows, d, st)) != PREDTOP_OK) return s;
  if ((s = embed_launch(m, dag, w.pe, w.x32, w.x16, st)) != PREDTOP_OK) return s;
  for (int l = 0; l <= last_layer; ++l) {
    const LayerDev& L = m->layer[l];
    GemmArgs a{};
    a.M = M; a.K = d; a.N = 3 * d; a.bias = L.bqkv; a.out16 = w.qkv;
    a.qcols = d;  // Q in log2 units for the attention kernel: q * log2(e) / sqrt(d_h)
    a.qscale = (float)(1.4426950408889634 / sqrt((double)(d / H)));
    {
      ProfScope _p(PK_GEMM_QKV, st);
      if ((s = gemm_launch(&tm_x16, &L.tm_qkv, m->bn_qkv, EPI_BIAS_F16, a, st)) != PREDTOP_OK) return s;
    }
    if ((s = attention_launch(dag, d, H, w.qkv, w.att, st)) != PREDTOP_OK) return s;
    if (use_fused_tail(d, f)) {
      ProfScope _p(PK_LAYER_TAIL, st);
      // after the last layer only the fp32 stream is read (readout, x_out):
      // the d = 256 tail skips its fp16 shadow there
      s = layer_tail256_supported(d, f) ? layer_tail256_launch(m, l, w.att, w.x32, l == last_layer ? nullptr : w.x16, M, st)
          : use_tail_v2(d, f)           ? layer_tail2_launch(m, l, w.att, w.x32, w.x16, M, st)
                                        : layer_tail_launch(m, l, w.att, w.x32, w.x16, M, st);
      if (s != PREDTOP_OK) return s;
      continue;
    }
    a = GemmArgs{};
    a.M = M; a.K = d; a.N = d; a.bias = L.bo; a.resid32 = w.x32; a.out32 = w.x32; a.out16 = w.x16;
    a.gamma = L.g1; a.beta = L.be1; a.eps = m->cfg.ln_eps;
    {
      ProfScope _p(PK_GEMM_O_LN, st);
      a.kch = ln32 ? 32 : 0;
      if ((s = gemm_launch(ln32 ? &tm_att32 : &tm_att, ln32 ? &L.tm_o32 : &L.tm_o, d, EPI_BIAS_RESID_LN, a, st)) !=
          PREDTOP_OK)
        return s;
    }
    a = GemmArgs{};
    a.M = M; a.K = d; a.N = f; a.bias = L.b1; a.out16 = w.hid;
    {
      ProfScope _p(PK_GEMM_FF1, st);
      if ((s = gemm_launch(&tm_x16, &L.tm_1, m->bn_ff1, EPI_BIAS_RELU_F16, a, st)) != PREDTOP_OK) return s;
    }
    a = GemmArgs{};
    a.M = M; a.K = f; a.N = d; a.bias = L.b2; a.resid32 = w.x32; a.out32 = w.x32; a.out16 = w.x16;
    a.gamma = L.g2; a.beta = L.be2; a.eps = m->cfg.ln_eps;
    {
      ProfScope _p(PK_GEMM_FF2_LN, st);
      a.kch = ln32 ? 32 : 0;
      if ((s = gemm_launch(ln32 ? &tm_hid32 : &tm_hid, ln32 ? &L.tm_2_32 : &L.tm_2, d, EPI_BIAS_RESID_LN, a, st)) !=
          PREDTOP_OK)
        return s;
    }
  }
  if (latency_out)
    if ((s = readout_launch(m, dag, w.x32, latency_out, st)) != PREDTOP_OK) return s;
  if (x_out)
    PT_CUDA_TRY(cudaMemcpyAsync(x_out, w.x32, sizeof(float) * (size_t)Ntot * d,
                                cudaMemcpyDeviceToDevice, st));
  return PREDTOP_OK;
}

predtop_status predtop_stage_forward(predtop_model model, predtop_dag dag, void* workspace,
                                     size_t ws_bytes, float* latency_out, void* cuda_stream) {
  if (!latency_out) { set_error("latency_out is NULL"); return PREDTOP_ERR_INVALID_ARG; }
  if (!model) { set_error("model is NULL"); return PREDTOP_ERR_INVALID_ARG; }
  return forward_impl(model, dag, workspace, ws_bytes, model->cfg.num_layers - 1, latency_out,
                      nullptr, S(cuda_stream));
}

predtop_status predtop_debug_node_embeddings(predtop_model model, predtop_dag dag, void* workspace,
                                             size_t ws_bytes, int32_t layer, float* x_out,
                                             void* cuda_stream) {
  if (!model || !x_out || layer < -1 || layer >= model->cfg.num_layers) {
    set_error("bad arguments");
    return PREDTOP_ERR_INVALID_ARG;
  }
  return forward_impl(model, dag, workspace, ws_bytes, layer, nullptr, x_out, S(cuda_stream));
}

// -------------------------------------------------------------------- plans
size_t predtop_plan_latency_workspace(void) { return 256; }

predtop_status predtop_plan_latency(int64_t num_plans, const int64_t* plan_ptr,
                                    const int32_t* plan_stage, const int32_t* microbatches,
                                    const float* stage_latency, int64_t num_stages, double* T_out,
                                    void* workspace, size_t ws_bytes, uint32_t flags,
                                    int64_t* first_bad_plan, void* cuda_stream) {
  if (first_bad_plan) *first_bad_plan = -1;
  if (num_plans < 0 || num_stages < 0) { set_error("negative size"); return PREDTOP_ERR_INVALID_ARG; }
  if (num_plans == 0) return PREDTOP_OK;
  if (!plan_ptr || !plan_stage || !microbatches || !T_out || !workspace ||
      (num_stages > 0 && !stage_latency)) {
    set_error("NULL argument");
    return PREDTOP_ERR_INVALID_ARG;
  }
  if (ws_bytes < predtop_plan_latency_workspace() || ((uintptr_t)workspace & 7)) {
    set_error("plan workspace too small");
    return PREDTOP_ERR_WORKSPACE;
  }
  int64_t* fb = (int64_t*)workspace;
  PT_CUDA_TRY(cudaMemsetAsync(fb, 0x7f, sizeof(int64_t), S(cuda_stream)));
  predtop_status s = plan_launch(num_plans, plan_ptr, plan_stage, microbatches, stage_latency,
                                 num_stages, T_out, fb, S(cuda_stream));
  if (s != PREDTOP_OK || (flags & PREDTOP_NO_SYNC)) return s;
  int64_t h = 0;
  PT_CUDA_TRY(cudaMemcpyAsync(&h, fb, sizeof(h), cudaMemcpyDeviceToHost, S(cuda_stream)));
  PT_CUDA_TRY(cudaStreamSynchronize(S(cuda_stream)));
  if (h >= 0 && h < num_plans) {
    if (first_bad_plan) *first_bad_plan = h;
    set_error("plan %lld is invalid", (long long)h);
    return PREDTOP_ERR_INVALID_ARG;
  }
  return PREDTOP_OK;
}

size_t predtop_plan_argmin_workspace(int64_t) { return 256; }

size_t predtop_prune_workspace(const predtop_batch_desc* desc) {
  DagBounds bd;
  if (!dag_bounds(desc, &bd)) return 0;
  return prune_workspace_bytes(desc);
}

predtop_status predtop_prune_graphs(const predtop_batch_desc* desc, const int64_t* node_ptr,
                                    const int64_t* edge_ptr, const int32_t* edge_src, const int32_t* edge_dst,
                                    const predtop_node_feat* feats, const uint16_t* pruned_ops,
                                    int32_t num_pruned_ops, void* workspace, size_t ws_bytes,
                                    int64_t* out_node_ptr, int64_t* out_edge_ptr, int32_t* out_src,
                                    int32_t* out_dst, int64_t edge_capacity, predtop_node_feat* out_feats,
                                    int64_t* totals, int32_t* first_bad_graph, void* cuda_stream) {
  if (first_bad_graph) *first_bad_graph = -1;
  DagBounds bd;
  if (!dag_bounds(desc, &bd)) { set_error("prune: invalid batch descriptor"); return PREDTOP_ERR_INVALID_ARG; }
  if (desc->max_nodes > PREDTOP_MAX_NODES) { set_error("prune: max_nodes too large"); return PREDTOP_ERR_TOO_LARGE; }
  if (!node_ptr || !edge_ptr || !feats || (desc->total_edges > 0 && (!edge_src || !edge_dst)) || !workspace ||
      !out_node_ptr || !out_edge_ptr || !out_feats || (edge_capacity > 0 && (!out_src || !out_dst)) ||
      !pruned_ops || num_pruned_ops < 1 || num_pruned_ops > PREDTOP_PRUNE_MAX_OPS || edge_capacity < 0) {
    set_error("prune: NULL or out-of-range argument");
    return PREDTOP_ERR_INVALID_ARG;
  }
  const size_t need = predtop_prune_workspace(desc);
  if (((uintptr_t)workspace & 255) || ws_bytes < need) {
    set_error("prune: workspace too small or misaligned (%zu < %zu)", ws_bytes, need);
    return PREDTOP_ERR_WORKSPACE;
  }
  if (!device_ok()) return PREDTOP_ERR_CUDA;
  return prune_launch(desc, node_ptr, edge_ptr, edge_src, edge_dst, feats, pruned_ops, num_pruned_ops, workspace,
                      out_node_ptr, out_edge_ptr, out_src, out_dst, edge_capacity, out_feats, totals,
                      first_bad_graph, S(cuda_stream));
}

size_t predtop_plan_search_workspace(int64_t num_problems, int32_t num_layers, int32_t num_choices) {
  if (num_problems < 1 || num_layers < 1 || num_layers > PREDTOP_SEARCH_MAX_LAYERS || num_choices < 1 ||
      num_choices > PREDTOP_SEARCH_MAX_CHOICES)
    return 0;
  return search_workspace_bytes(num_problems, num_layers, num_choices);
}

predtop_status predtop_plan_search(int64_t num_problems, int32_t num_layers, int32_t num_choices,
                                   const int32_t* choice_devices, int32_t num_devices,
                                   const float* stage_latency, int64_t table_stride, int64_t num_tables,
                                   const int32_t* problem_table, const int32_t* microbatches,
                                   double* T_out, int32_t* num_stages_out, int32_t* stage_end_out,
                                   int32_t* stage_choice_out, void* workspace, size_t ws_bytes,
                                   void* cuda_stream) {
  const size_t need = predtop_plan_search_workspace(num_problems, num_layers, num_choices);
  if (need == 0) {
    set_error("plan_search: bad sizes (P=%lld L=%d K=%d)", (long long)num_problems, num_layers, num_choices);
    return PREDTOP_ERR_INVALID_ARG;
  }
  if (table_stride < (int64_t)num_layers * (num_layers + 1) / 2) {
    set_error("plan_search: table_stride %lld < L(L+1)/2", (long long)table_stride);
    return PREDTOP_ERR_INVALID_ARG;
  }
  if (num_devices < 1 || num_devices > PREDTOP_SEARCH_MAX_DEVICES || num_tables < 1) {
    set_error("plan_search: num_devices %d / num_tables %lld out of range", num_devices, (long long)num_tables);
    return PREDTOP_ERR_INVALID_ARG;
  }
  if (!choice_devices || !stage_latency || !microbatches || !T_out || !num_stages_out || !stage_end_out ||
      !stage_choice_out || !workspace) {
    set_error("plan_search: NULL argument");
    return PREDTOP_ERR_INVALID_ARG;
  }
  for (int c = 0; c < num_choices; ++c)
    if (choice_devices[c] < 1) { set_error("plan_search: choice_devices[%d] < 1", c); return PREDTOP_ERR_INVALID_ARG; }
  if (((uintptr_t)workspace & 255) || ws_bytes < need) {
    set_error("plan_search: workspace too small or misaligned (%zu < %zu)", ws_bytes, need);
    return PREDTOP_ERR_WORKSPACE;
  }
  if (!device_ok()) return PREDTOP_ERR_CUDA;
  return search_launch(num_problems, num_layers, num_choices, choice_devices, num_devices, stage_latency,
                       table_stride, num_tables, problem_table, microbatches, T_out, num_stages_out, stage_end_out,
                       stage_choice_out, workspace, S(cuda_stream));
}

predtop_status predtop_plan_argmin(int64_t num_plans, const double* T, int64_t* best_out,
                                   void* workspace, size_t ws_bytes, void* cuda_stream) {
  (void)workspace;
  (void)ws_bytes;
  if (num_plans < 0 || !best_out || (num_plans > 0 && !T)) {
    set_error("bad arguments");
    return PREDTOP_ERR_INVALID_ARG;
  }
  return argmin_launch(num_plans, T, best_out, S(cuda_stream));
}

}  // extern "C"
