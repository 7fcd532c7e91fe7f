"""Python front-end of the CPU fp64 oracle (oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / --impl reference leg, never by the product package.
It shares no code with the CUDA path; it only reads the synthetic inputs of
paper_conf_ipps_acharyas25_b200.synth (a generator with no method arithmetic).

All arithmetic happens in oracle.c; this module marshals numpy arrays.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading
from concurrent.futures import ThreadPoolExecutor
from typing import Dict, List, Optional, Sequence

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "oracle.c")
LIB = os.path.join(HERE, "liboracle.so")

OK, RANGE, SELF_LOOP, CYCLE = 0, -2, -3, -4
F = 80
FEAT_DTYPE = np.dtype([("op", "<u2"), ("dtype", "u1"), ("kind", "u1"), ("dims", "<u4", (4,))])

_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (-ffp-contract=off: no FMA contraction)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < max(
            os.path.getmtime(SRC), os.path.getmtime(os.path.join(HERE, "oracle.h"))):
        tmp = LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
                               "-shared", "-Wall", "-o", tmp, SRC, "-lm"])
        os.replace(tmp, LIB)
    return LIB


class _Cfg(ctypes.Structure):
    _fields_ = [("L", ctypes.c_int), ("d", ctypes.c_int), ("H", ctypes.c_int),
                ("d_ff", ctypes.c_int), ("pool", ctypes.c_int), ("ln_eps", ctypes.c_double)]


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(LIB)
            P = ctypes.c_void_p
            i32, i64, dbl = ctypes.c_int, ctypes.c_int64, ctypes.c_double
            L.orc_validate.argtypes = [i32, i32, P, P]
            L.orc_validate.restype = i32
            L.orc_depth.argtypes = [i32, i32, P, P, P]
            L.orc_row_words.argtypes = [i32]
            L.orc_row_words.restype = i32
            L.orc_reach.argtypes = [i32, i32, P, P, P]
            L.orc_reach_k.argtypes = [i32, i32, P, P, i32, P]
            L.orc_mask.argtypes = [i32, P, P]
            L.orc_tiles.argtypes = [i32, P, P]
            L.orc_tiles.restype = i64
            L.orc_blob_floats.argtypes = [P]
            L.orc_blob_floats.restype = ctypes.c_long
            L.orc_features.argtypes = [i32, P, P]
            L.orc_embed.argtypes = [P, P, i32, P, P, P]
            L.orc_attention.argtypes = [P, P, i32, i32, P, P, P]
            L.orc_layer.argtypes = [P, P, i32, i32, P, P, P]
            L.orc_qkv_rows.argtypes = [P, P, i32, i32, i32, P, P]
            L.orc_attention_rows.argtypes = [P, i32, P, P, i32, i32, P]
            L.orc_layer_post_rows.argtypes = [P, P, i32, i32, i32, P, P, P]
            L.orc_readout.argtypes = [P, P, i32, P]
            L.orc_readout.restype = dbl
            L.orc_forward.argtypes = [P, P, i32, i32, P, P, P, P, P]
            L.orc_forward.restype = i32
            L.orc_forward_k.argtypes = [P, P, i32, i32, P, P, P, i32, P, P]
            L.orc_forward_k.restype = i32
            L.orc_plan_T.argtypes = [i64, P, P, P, P, i64, P]
            L.orc_argmin.argtypes = [i64, P]
            L.orc_argmin.restype = i64
            L.orc_prune.argtypes = [i32, i32, P, P, P, P, i32, P, P, P, P, P]
            L.orc_prune.restype = i32
            L.orc_plan_search.argtypes = [i32, i32, P, i32, P, i32, P, P, P]
            L.orc_plan_search.restype = dbl
            L.orc_grad.argtypes = [P, P, i32, i32, P, P, P, dbl, P, P]
            L.orc_grad.restype = i32
            _lib = L
    return _lib


def _p(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _i32(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.int32)


def _feats(f) -> np.ndarray:
    return np.ascontiguousarray(f, dtype=FEAT_DTYPE)


def cfg(model_cfg: dict) -> _Cfg:
    return _Cfg(model_cfg["num_layers"], model_cfg["d_model"], model_cfg["num_heads"],
                model_cfg["d_ff"], model_cfg.get("pool", 0), float(model_cfg.get("ln_eps", 1e-5)))


# ---- graph steps -----------------------------------------------------------
def validate(n, src, dst) -> int:
    s, d = _i32(src), _i32(dst)
    return lib().orc_validate(n, len(s), _p(s), _p(d))


def depth(n, src, dst) -> np.ndarray:
    s, d = _i32(src), _i32(dst)
    out = np.zeros(n, np.int32)
    lib().orc_depth(n, len(s), _p(s), _p(d), _p(out))
    return out


def row_words(n: int) -> int:
    return 2 * ((n + 127) // 128)


def reach(n, src, dst, hops: int = 0) -> np.ndarray:
    """Closure bitsets [n, W] uint64 (layout of include/predtop.h).  hops > 0:
    the k-hop relation R_k (finite-k DAGRA, reading R19)."""
    s, d = _i32(src), _i32(dst)
    out = np.zeros((n, row_words(n)), np.uint64)
    if hops > 0:
        lib().orc_reach_k(n, len(s), _p(s), _p(d), int(hops), _p(out))
    else:
        lib().orc_reach(n, len(s), _p(s), _p(d), _p(out))
    return out


def mask(n, R: np.ndarray) -> np.ndarray:
    R = np.ascontiguousarray(R, np.uint64)
    out = np.zeros_like(R)
    lib().orc_mask(n, _p(R), _p(out))
    return out


def tiles(n, M: np.ndarray):
    M = np.ascontiguousarray(M, np.uint64)
    T = (n + 127) // 128
    cls = np.zeros(T * T, np.uint8)
    pairs = lib().orc_tiles(n, _p(M), _p(cls))
    return cls, int(pairs)


def bits_to_dense(B: np.ndarray, n: int) -> np.ndarray:
    """[n, W] uint64 bitset rows -> dense bool [n, n] (bit u%64 of word u/64)."""
    by = np.ascontiguousarray(B).view(np.uint8).reshape(B.shape[0], -1)
    return np.unpackbits(by, axis=1, bitorder="little")[:, :n].astype(bool)


# ---- model steps -----------------------------------------------------------
def blob_floats(model_cfg) -> int:
    c = cfg(model_cfg)
    return lib().orc_blob_floats(ctypes.byref(c))


def features(n, feats) -> np.ndarray:
    f = _feats(feats)
    out = np.zeros((n, F), np.float64)
    lib().orc_features(n, _p(f), _p(out))
    return out


def embed(model_cfg, blob, n, feats, dep) -> np.ndarray:
    c = cfg(model_cfg)
    b = np.ascontiguousarray(blob, np.float32)
    out = np.zeros((n, model_cfg["d_model"]), np.float64)
    lib().orc_embed(ctypes.byref(c), _p(b), n, _p(_feats(feats)), _p(_i32(dep)), _p(out))
    return out


def attention(model_cfg, blob, layer, n, M, x) -> np.ndarray:
    c = cfg(model_cfg)
    b = np.ascontiguousarray(blob, np.float32)
    x = np.ascontiguousarray(x, np.float64)
    out = np.zeros((n, model_cfg["d_model"]), np.float64)
    lib().orc_attention(ctypes.byref(c), _p(b), layer, n, _p(np.ascontiguousarray(M, np.uint64)),
                        _p(x), _p(out))
    return out


def layer(model_cfg, blob, li, n, M, x) -> np.ndarray:
    c = cfg(model_cfg)
    b = np.ascontiguousarray(blob, np.float32)
    x = np.ascontiguousarray(x, np.float64)
    out = np.zeros_like(x)
    lib().orc_layer(ctypes.byref(c), _p(b), li, n, _p(np.ascontiguousarray(M, np.uint64)),
                    _p(x), _p(out))
    return out


def readout(model_cfg, blob, n, x) -> float:
    c = cfg(model_cfg)
    b = np.ascontiguousarray(blob, np.float32)
    return float(lib().orc_readout(ctypes.byref(c), _p(b), n, _p(np.ascontiguousarray(x, np.float64))))


def forward(model_cfg, blob, n, src, dst, feats, taps: bool = False, hops: int = 0):
    """One stage graph -> (status, latency, taps or None).  hops > 0: k-hop mask."""
    c = cfg(model_cfg)
    b = np.ascontiguousarray(blob, np.float32)
    s, d = _i32(src), _i32(dst)
    y = np.zeros(1, np.float64)
    t = np.zeros((model_cfg["num_layers"] + 1, n, model_cfg["d_model"]), np.float64) if taps else None
    st = lib().orc_forward_k(ctypes.byref(c), _p(b), n, len(s), _p(s), _p(d), _p(_feats(feats)),
                             int(hops), _p(y), _p(t))
    return st, float(y[0]), t


def forward_batch(model_cfg, blob, batch, graphs: Optional[Sequence[int]] = None,
                  threads: Optional[int] = None, hops: int = 0) -> np.ndarray:
    """Latency of every graph (or the listed ones) of a synth.StageBatch, one
    graph per worker thread (ctypes releases the GIL)."""
    gs = list(range(batch.num_graphs)) if graphs is None else list(graphs)
    threads = threads or (os.cpu_count() or 1)
    lib()

    def one(g):
        n, s, d, f = batch.graph(g)
        return forward(model_cfg, blob, n, s, d, f, hops=hops)[1]

    if threads <= 1 or len(gs) <= 1:
        return np.asarray([one(g) for g in gs], np.float64)
    with ThreadPoolExecutor(threads) as ex:
        return np.asarray(list(ex.map(one, gs)), np.float64)


def head_condition(model_cfg, blob, n, x_final) -> float:
    """Condition scale of the head's last dot product (reading R10):
    sum_i |w_o,i * h2_i| with h2 = ReLU(H_2 ReLU(H_1 g + c_1) + c_2) and g
    the pooled final embeddings (Eqn 2).  It is the magnitude of the
    terms that cancel in y - c_o = w_o . h2, so |dy| / head_condition is the
    normwise relative error of the computed (bias-free) part (reading R22);
    dividing by |y - c_o| instead is ill-conditioned where the terms cancel.
    Test metadata only: numpy on the oracle's own fp64 taps, the blob's head
    weights in the include/predtop.h order (H_1, c_1, H_2, c_2, w_o, c_o last)."""
    d = model_cfg["d_model"]
    b = np.asarray(blob, np.float64)
    tail = b[len(b) - (2 * d * d + 3 * d + 1):]
    H1 = tail[:d * d].reshape(d, d)
    c1 = tail[d * d:d * d + d]
    H2 = tail[d * d + d:2 * d * d + d].reshape(d, d)
    c2 = tail[2 * d * d + d:2 * d * d + 2 * d]
    wo = tail[2 * d * d + 2 * d:2 * d * d + 3 * d]
    g = np.asarray(x_final, np.float64).sum(0)
    if model_cfg.get("pool", 0) == 1:
        g = g / n
    h1 = np.maximum(H1 @ g + c1, 0.0)
    h2 = np.maximum(H2 @ h1 + c2, 0.0)
    return float(np.abs(wo * h2).sum())


def forward_batch_cond(model_cfg, blob, batch, graphs: Optional[Sequence[int]] = None,
                       threads: Optional[int] = None, hops: int = 0):
    """(latency, head_condition) of every listed graph: forward_batch plus the
    condition scale of each graph's bias-free output (from its final taps)."""
    gs = list(range(batch.num_graphs)) if graphs is None else list(graphs)
    threads = threads or (os.cpu_count() or 1)
    lib()

    def one(g):
        n, s, d, f = batch.graph(g)
        _, y, t = forward(model_cfg, blob, n, s, d, f, taps=True, hops=hops)
        return y, head_condition(model_cfg, blob, n, t[-1])

    if threads <= 1 or len(gs) <= 1:
        out = [one(g) for g in gs]
    else:
        with ThreadPoolExecutor(threads) as ex:
            out = list(ex.map(one, gs))
    return np.asarray([o[0] for o in out], np.float64), np.asarray([o[1] for o in out], np.float64)


# ---- training ------------------------------------
def grad(model_cfg, blob, n, src, dst, feats, dy: float = 1.0, out: Optional[np.ndarray] = None):
    """(y, grad): latency of one graph and dy * d y / d theta over the weight
    blob (orc_grad, fp64; accumulated into `out` when given)."""
    c = cfg(model_cfg)
    b = np.ascontiguousarray(blob, np.float32)
    s, d = _i32(src), _i32(dst)
    g = np.zeros(len(b), np.float64) if out is None else out
    y = np.zeros(1, np.float64)
    st = lib().orc_grad(ctypes.byref(c), _p(b), n, len(s), _p(s), _p(d), _p(_feats(feats)), float(dy), _p(y), _p(g))
    if st != OK:
        raise ValueError(f"invalid graph (status {st})")
    return float(y[0]), g


def mae_grad(model_cfg, blob, batch, y_true, threads: Optional[int] = None):
    """Eqn 3: L = (1/N) sum_i |y_hat_i - y_i| over the graphs of a
    synth.StageBatch, and dL/dtheta = sum_i sign(y_hat_i - y_i)/N * dy_hat_i/dtheta
    (sign(0) = 0).  Returns (L, grad, y_hat).  Two passes: the forward latencies
    (forward_batch) fix the signs, then orc_grad per graph."""
    y_true = np.asarray(y_true, np.float64)
    N = batch.num_graphs
    y_hat = forward_batch(model_cfg, blob, batch, threads=threads)
    loss = float(np.mean(np.abs(y_hat - y_true)))
    sgn = np.sign(y_hat - y_true) / N
    threads = threads or (os.cpu_count() or 1)
    parts = [np.zeros(len(blob), np.float64) for _ in range(min(threads, N))]

    def one(i):
        g = i % len(parts)
        n, s, d, f = batch.graph(i)
        return g, grad(model_cfg, blob, n, s, d, f, dy=sgn[i])[1]

    total = np.zeros(len(blob), np.float64)
    with ThreadPoolExecutor(threads) as ex:
        for _, gi in ex.map(one, range(N)):
            total += gi
    return loss, total, y_hat


def adam_step(param, grad_, m, v, step: int, lr: float, beta1: float = 0.9, beta2: float = 0.999,
              eps: float = 1e-8):
    """One Adam update (PyTorch's Adam with its defaults), written out
    as torch.optim.Adam computes it (no weight decay, amsgrad off), fp64:
      m = b1 m + (1-b1) g;  v = b2 v + (1-b2) g^2;
      p -= lr / (1 - b1^t) * m / (sqrt(v) / sqrt(1 - b2^t) + eps).
    Returns new (param, m, v)."""
    g = np.asarray(grad_, np.float64)
    m = beta1 * np.asarray(m, np.float64) + (1.0 - beta1) * g
    v = beta2 * np.asarray(v, np.float64) + (1.0 - beta2) * g * g
    bc1 = 1.0 - beta1 ** step
    bc2 = 1.0 - beta2 ** step
    denom = np.sqrt(v) / np.sqrt(bc2) + eps
    p = np.asarray(param, np.float64) - (lr / bc1) * m / denom
    return p, m, v


def cosine_lr(epoch: int, epochs: int, lr0: float = 1e-3) -> float:
    """Cosine decay: lr0 in the first epoch down to 0 in the last,
    lr_e = lr0 * (1 + cos(pi * e / (E - 1))) / 2 for e = 0 .. E-1."""
    if epochs <= 1:
        return lr0
    return lr0 * 0.5 * (1.0 + np.cos(np.pi * epoch / (epochs - 1)))


# ---- one large graph, row block by row block --------------------------------
def _ranges(rows, threads):
    """Split a sorted row list into <= ~4*threads contiguous runs."""
    rows = np.asarray(rows, np.int64)
    runs, a = [], 0
    for i in range(1, len(rows) + 1):
        if i == len(rows) or rows[i] != rows[i - 1] + 1:
            runs.append((int(rows[a]), int(rows[i - 1]) + 1))
            a = i
    out = []
    target = max(1, len(rows) // max(1, 4 * threads))
    for r0, r1 in runs:
        for b in range(r0, r1, target):
            out.append((b, min(r1, b + target)))
    return out


def layer_rows(model_cfg, blob, li, n, M, x, rows=None, threads=None) -> np.ndarray:
    """orc_layer for one graph evaluated row block by row block on `threads`
    workers, from the same pieces orc_layer composes (orc_qkv_rows for every
    row, orc_attention_rows and orc_layer_post_rows for the requested rows).
    rows: None = all rows (returns [n, d]); else a sorted subset (returns
    [len(rows), d])."""
    L = lib()
    c = cfg(model_cfg)
    d = model_cfg["d_model"]
    threads = threads or (os.cpu_count() or 1)
    b = np.ascontiguousarray(blob, np.float32)
    x = np.ascontiguousarray(x, np.float64)
    M = np.ascontiguousarray(M, np.uint64)
    qkv = np.zeros((n, 3 * d), np.float64)
    a = np.zeros((n, d), np.float64)
    out = np.zeros((n, d), np.float64)
    sel = np.arange(n) if rows is None else np.asarray(sorted(rows), np.int64)
    with ThreadPoolExecutor(threads) as ex:
        list(ex.map(lambda r: L.orc_qkv_rows(ctypes.byref(c), _p(b), li, r[0], r[1], _p(x), _p(qkv)),
                    _ranges(np.arange(n), threads)))
        blocks = _ranges(sel, threads)
        list(ex.map(lambda r: L.orc_attention_rows(ctypes.byref(c), n, _p(M), _p(qkv), r[0], r[1], _p(a)), blocks))
        list(ex.map(lambda r: L.orc_layer_post_rows(ctypes.byref(c), _p(b), li, r[0], r[1], _p(a), _p(x), _p(out)),
                    blocks))
    return out if rows is None else out[sel]


def forward_rows(model_cfg, blob, n, src, dst, feats, threads=None, taps: bool = False, timings=None):
    """orc_forward for ONE (large) graph with every layer evaluated row block
    by row block in parallel (layer_rows); the graph steps (validate, depth,
    reach, mask), embedding and readout are the single-threaded oracle calls.
    Returns (status, latency, taps or None); `timings` (dict) gets the wall
    seconds of the graph steps and of each layer."""
    import time
    t0 = time.perf_counter()
    st = validate(n, src, dst)
    if st != OK:
        return st, float("nan"), None
    dep = depth(n, src, dst)
    R = reach(n, src, dst)
    M = mask(n, R)
    t1 = time.perf_counter()
    x = embed(model_cfg, blob, n, feats, dep)
    tp = [x] if taps else None
    lt = []
    for li in range(model_cfg["num_layers"]):
        a = time.perf_counter()
        x = layer_rows(model_cfg, blob, li, n, M, x, threads=threads)
        lt.append(time.perf_counter() - a)
        if taps:
            tp.append(x)
    y = readout(model_cfg, blob, n, x)
    if timings is not None:
        timings.update({"graph_steps_s": t1 - t0, "layers_s": lt, "total_s": time.perf_counter() - t0})
    return OK, y, (np.stack(tp) if taps else None)


# ---- pipeline formula ------------------------------------------------------
def plan_T(plan_ptr, plan_stage, microbatches, stage_latency) -> np.ndarray:
    pp = np.ascontiguousarray(plan_ptr, np.int64)
    ps = np.ascontiguousarray(plan_stage, np.int32)
    B = np.ascontiguousarray(microbatches, np.int32)
    t = np.ascontiguousarray(stage_latency, np.float32)
    T = np.zeros(len(pp) - 1, np.float64)
    lib().orc_plan_T(len(pp) - 1, _p(pp), _p(ps), _p(B), _p(t), len(t), _p(T))
    return T


def argmin(T) -> int:
    T = np.ascontiguousarray(T, np.float64)
    return int(lib().orc_argmin(len(T), _p(T)))


def plan_search(stage_latency, choice_devices, num_devices: int, microbatches: int):
    """Optimal pipeline plan over a stage table t[L][L][K] (fp32; entries with
    i > j unused; non-finite or negative = infeasible) by exhaustive
    enumeration (reading R20) -> (T*, [(first, last, choice), ...])."""
    t = np.ascontiguousarray(stage_latency, np.float32)
    L, L2, K = t.shape
    assert L == L2
    dev = np.ascontiguousarray(choice_devices, np.int32)
    S = ctypes.c_int32(0)
    ends = np.zeros(64, np.int32)
    ch = np.zeros(64, np.int32)
    T = lib().orc_plan_search(L, K, _p(dev), int(num_devices), _p(t), int(microbatches),
                              ctypes.byref(S), _p(ends), _p(ch))
    stages, a = [], 0
    for i in range(S.value):
        stages.append((a, int(ends[i]), int(ch[i])))
        a = int(ends[i]) + 1
    return float(T), stages


def prune(n, src, dst, feats, ops=(64, 65)):
    """Graph pruning (SIV-B4; reading R21) -> (status, nk, src', dst', feats')."""
    s, d, f = _i32(src), _i32(dst), _feats(feats)
    o = np.ascontiguousarray(ops, np.uint16)
    nk = ctypes.c_int32(0)
    ne = ctypes.c_int64(0)
    cap = max(1, n * n)
    os_ = np.zeros(cap, np.int32)
    od = np.zeros(cap, np.int32)
    of = np.zeros(max(n, 1), FEAT_DTYPE)
    st = lib().orc_prune(n, len(s), _p(s), _p(d), _p(f), _p(o), len(o), ctypes.byref(nk), _p(os_), _p(od),
                         ctypes.byref(ne), _p(of))
    if st != OK:
        return st, 0, None, None, None
    return st, nk.value, os_[:ne.value].copy(), od[:ne.value].copy(), of[:nk.value].copy()
