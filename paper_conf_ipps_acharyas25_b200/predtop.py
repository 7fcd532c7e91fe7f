"""Thin ctypes binding of libpredtop (include/predtop.h).

Argument marshalling only: every step of the prediction path runs in the
library's sm_100a kernels.  torch provides device memory and streams.  There
is no CPU fallback: if the library or a CUDA device is missing, calls raise.

Low-level functions keep the C names (predtop_build_dag, predtop_reachability,
predtop_stage_forward, predtop_plan_latency, ...); the small classes below
(DeviceBatch, Dag, Model) own the torch buffers those calls need.
"""
from __future__ import annotations

import ctypes
import os
import threading
from typing import Optional

import numpy as np
import torch

from . import build as _build

PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("PREDTOP_LIB", _build.LIB)  # override: debug builds (tools/)

OK, INVALID_ARG, RANGE, SELF_LOOP, CYCLE, TOO_LARGE, WORKSPACE, CUDA, UNSUPPORTED = \
    0, -1, -2, -3, -4, -5, -6, -7, -8
NO_SYNC = 1
POOL_SUM, POOL_MEAN = 0, 1
MAX_NODES = 65536
MAX_PLAN_STAGES = 64
SEARCH_MAX_LAYERS, SEARCH_MAX_CHOICES, SEARCH_MAX_DEVICES = 64, 32, 64
OP_RESHAPE, OP_CONVERT_ELEMENT_TYPE = 64, 65


class PredtopError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"predtop status {status}: {msg}")
        self.status = status


class BatchDesc(ctypes.Structure):
    _fields_ = [("num_graphs", ctypes.c_int32), ("max_nodes", ctypes.c_int32),
                ("total_nodes", ctypes.c_int64), ("total_edges", ctypes.c_int64),
                ("flags", ctypes.c_uint32), ("hops", ctypes.c_int32)]


class ModelConfig(ctypes.Structure):
    _fields_ = [("num_layers", ctypes.c_int32), ("d_model", ctypes.c_int32),
                ("num_heads", ctypes.c_int32), ("d_ff", ctypes.c_int32),
                ("pool", ctypes.c_int32), ("ln_eps", ctypes.c_float)]


_lib = None
_lock = threading.Lock()
_P, _I32, _I64, _U32, _SZ = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32, ctypes.c_size_t

_SIGS = {
    "predtop_build_dag_workspace": (_SZ, [_P]),
    "predtop_build_dag": (_I32, [_P, _P, _P, _P, _P, _P, _P, _SZ, _P, _P, _P, _P]),
    "predtop_dag_status": (_I32, [_P, _P, _P]),
    "predtop_dag_reach_words": (_I32, [_P, _P, _P]),
    "predtop_reachability": (_I32, [_P, _P, _P]),
    "predtop_debug_mask": (_I32, [_P, _P, _P]),
    "predtop_debug_tiles": (_I32, [_P, _P, _P, _P]),
    "predtop_dag_destroy": (None, [_P]),
    "predtop_model_weight_floats": (_SZ, [_P]),
    "predtop_model_device_bytes": (_SZ, [_P]),
    "predtop_model_create": (_I32, [_P, _P, _SZ, _P, _SZ, _P]),
    "predtop_model_destroy": (None, [_P]),
    "predtop_stage_forward_workspace": (_SZ, [_P, _P]),
    "predtop_stage_forward": (_I32, [_P, _P, _P, _SZ, _P, _P]),
    "predtop_debug_node_embeddings": (_I32, [_P, _P, _P, _SZ, _I32, _P, _P]),
    "predtop_plan_latency_workspace": (_SZ, []),
    "predtop_plan_latency": (_I32, [_I64, _P, _P, _P, _P, _I64, _P, _P, _SZ, _U32, _P, _P]),
    "predtop_plan_argmin_workspace": (_SZ, [_I64]),
    "predtop_plan_argmin": (_I32, [_I64, _P, _P, _P, _SZ, _P]),
    "predtop_prune_workspace": (_SZ, [_P]),
    "predtop_prune_graphs": (_I32, [_P, _P, _P, _P, _P, _P, _P, _I32, _P, _SZ, _P, _P, _P, _P, _I64, _P, _P, _P, _P]),
    "predtop_plan_search_workspace": (_SZ, [_I64, _I32, _I32]),
    "predtop_plan_search": (_I32, [_I64, _I32, _I32, _P, _I32, _P, _I64, _I64, _P, _P, _P, _P, _P, _P, _P, _SZ, _P]),
    "predtop_train_state_bytes": (_SZ, [_P]),
    "predtop_train_create": (_I32, [_P, _P, _SZ, _P, _SZ, _P]),
    "predtop_train_destroy": (None, [_P]),
    "predtop_train_workspace": (_SZ, [_P, _P]),
    "predtop_train_grad": (_I32, [_P, _P, _P, _P, _SZ, _P, _P, _P]),
    "predtop_train_adam": (_I32, [_P, ctypes.c_float, _I32, ctypes.c_float, ctypes.c_float, ctypes.c_float, _P]),
    "predtop_train_buffer": (_P, [_P, _I32]),
    "predtop_status_string": (ctypes.c_char_p, [_I32]),
    "predtop_last_error": (ctypes.c_char_p, []),
    "predtop_abi_version": (ctypes.c_int, []),
    "predtop_launch_count": (_I64, []),
    "predtop_profile_enable": (None, [ctypes.c_int]),
    "predtop_profile_read": (ctypes.c_int, [_P, _P, ctypes.c_int]),
    "predtop_profile_kind_name": (ctypes.c_char_p, [ctypes.c_int]),
}


def lib():
    """Load libpredtop.so (built in-tree by build.py).  Raises if it is missing:
    there is no fallback path."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise RuntimeError(f"{LIB_PATH} is not built (run __graft_entry__.build())")
            L = ctypes.CDLL(LIB_PATH)
            for name, (res, args) in _SIGS.items():
                f = getattr(L, name)
                f.restype = res
                f.argtypes = args
            _lib = L
    return _lib


def _check(status: int):
    if status != OK:
        raise PredtopError(status, lib().predtop_last_error().decode(errors="replace"))


def _ptr(t: Optional[torch.Tensor]):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _stream(stream=None):
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def launch_count() -> int:
    return int(lib().predtop_launch_count())


# --------------------------------------------------------------- raw C names
def predtop_build_dag(desc: BatchDesc, node_ptr, edge_ptr, src, dst, feats, workspace,
                      depth_out=None, stream=None):
    h = ctypes.c_void_p()
    bad = ctypes.c_int32(-1)
    st = lib().predtop_build_dag(ctypes.byref(desc), _ptr(node_ptr), _ptr(edge_ptr), _ptr(src),
                                 _ptr(dst), _ptr(feats), _ptr(workspace), workspace.numel(),
                                 _ptr(depth_out), ctypes.byref(h), ctypes.byref(bad), _stream(stream))
    return st, h, bad.value


def predtop_reachability(dag_handle, bits_out: torch.Tensor, stream=None):
    _check(lib().predtop_reachability(dag_handle, _ptr(bits_out), _stream(stream)))


def predtop_stage_forward(model_handle, dag_handle, workspace: torch.Tensor, latency_out: torch.Tensor,
                          stream=None):
    _check(lib().predtop_stage_forward(model_handle, dag_handle, _ptr(workspace), workspace.numel(),
                                       _ptr(latency_out), _stream(stream)))


def predtop_plan_latency(plan_ptr, plan_stage, microbatches, stage_latency, T_out, workspace,
                         flags=0, stream=None):
    """Eqn 4 for every plan; returns (status, first bad plan or -1)."""
    bad = ctypes.c_int64(-1)
    st = lib().predtop_plan_latency(plan_ptr.numel() - 1, _ptr(plan_ptr), _ptr(plan_stage),
                                    _ptr(microbatches), _ptr(stage_latency), stage_latency.numel(),
                                    _ptr(T_out), _ptr(workspace), workspace.numel(), flags,
                                    ctypes.byref(bad), _stream(stream))
    if st != OK and st != INVALID_ARG:
        _check(st)
    return st, bad.value


def predtop_plan_argmin(T: torch.Tensor, best_out: torch.Tensor, stream=None):
    _check(lib().predtop_plan_argmin(T.numel(), _ptr(T), _ptr(best_out), None, 0, _stream(stream)))


# ------------------------------------------------------------ owning wrappers
FEAT_BYTES = 20


class DeviceBatch:
    """A packed batch of stage DAGs resident on the device (synth.StageBatch layout)."""

    def __init__(self, node_ptr, edge_ptr, src, dst, feats_bytes, max_nodes: int):
        self.node_ptr, self.edge_ptr, self.src, self.dst, self.feats = node_ptr, edge_ptr, src, dst, feats_bytes
        self.max_nodes = int(max_nodes)
        self.num_graphs = node_ptr.numel() - 1
        self.total_nodes = feats_bytes.numel() // FEAT_BYTES
        self.total_edges = src.numel()

    @staticmethod
    def from_host(batch, device="cuda", pin: bool = False) -> "DeviceBatch":
        def t(a, dtype):
            x = torch.from_numpy(np.ascontiguousarray(a)).to(dtype)
            return x.to(device, non_blocking=pin) if not pin else x.pin_memory().to(device, non_blocking=True)
        fb = np.ascontiguousarray(batch.feats).view(np.uint8).reshape(-1)
        sizes = np.diff(batch.node_ptr)
        return DeviceBatch(t(batch.node_ptr, torch.int64), t(batch.edge_ptr, torch.int64),
                           t(batch.src, torch.int32), t(batch.dst, torch.int32),
                           torch.from_numpy(fb.copy()).to(device), int(sizes.max()) if len(sizes) else 1)

    def desc(self, flags=0, hops: int = 0) -> BatchDesc:
        """hops: DAGRA range k (0 = infinity); k >= 1 builds the k-hop mask."""
        return BatchDesc(self.num_graphs, self.max_nodes, self.total_nodes, self.total_edges, flags, hops)


class Dag:
    """predtop_build_dag over a DeviceBatch; owns the workspace and depth."""

    def __init__(self, batch: DeviceBatch, no_sync: bool = False, stream=None, check: bool = True,
                 workspace: Optional[torch.Tensor] = None, depth: Optional[torch.Tensor] = None,
                 hops: int = 0):
        self.batch = batch
        dev = batch.node_ptr.device
        self.desc = batch.desc(NO_SYNC if no_sync else 0, hops)
        need = lib().predtop_build_dag_workspace(ctypes.byref(self.desc))
        if need == 0:
            raise PredtopError(INVALID_ARG, "invalid batch descriptor")
        self.workspace = workspace if workspace is not None and workspace.numel() >= need else \
            torch.empty(need, dtype=torch.uint8, device=dev)
        self.depth = depth if depth is not None else torch.empty(max(batch.total_nodes, 1), dtype=torch.int32, device=dev)
        self.status, self.handle, self.first_bad = predtop_build_dag(
            self.desc, batch.node_ptr, batch.edge_ptr, batch.src, batch.dst, batch.feats,
            self.workspace, self.depth, stream)
        if self.handle.value is None:
            _check(self.status)
        if check and self.status not in (OK,) and self.status not in (RANGE, SELF_LOOP, CYCLE, TOO_LARGE):
            _check(self.status)

    def rebuild(self, stream=None):
        """Re-run the device build on the same buffers (same shapes, new contents)."""
        lib().predtop_dag_destroy(self.handle)
        self.status, self.handle, self.first_bad = predtop_build_dag(
            self.desc, self.batch.node_ptr, self.batch.edge_ptr, self.batch.src, self.batch.dst,
            self.batch.feats, self.workspace, self.depth, stream)
        return self.status

    def dag_status(self, stream=None):
        bad = ctypes.c_int32(-1)
        st = lib().predtop_dag_status(self.handle, ctypes.byref(bad), _stream(stream))
        return st, bad.value

    def reach_words(self, stream=None) -> int:
        w = ctypes.c_int64(0)
        _check(lib().predtop_dag_reach_words(self.handle, ctypes.byref(w), _stream(stream)))
        return w.value

    def reachability(self, stream=None) -> torch.Tensor:
        out = torch.zeros(max(self.reach_words(stream), 1), dtype=torch.int64, device=self.workspace.device)
        predtop_reachability(self.handle, out, stream)
        return out

    def mask(self, stream=None) -> torch.Tensor:
        out = torch.zeros(max(self.reach_words(stream), 1), dtype=torch.int64, device=self.workspace.device)
        _check(lib().predtop_debug_mask(self.handle, _ptr(out), _stream(stream)))
        return out

    def tiles(self, num_tiles: int, stream=None):
        dev = self.workspace.device
        cls = torch.zeros(max(num_tiles, 1), dtype=torch.uint8, device=dev)
        pairs = torch.zeros(self.batch.num_graphs, dtype=torch.int64, device=dev)
        _check(lib().predtop_debug_tiles(self.handle, _ptr(cls), _ptr(pairs), _stream(stream)))
        return cls, pairs

    def __del__(self):
        try:
            if self.handle and self.handle.value:
                lib().predtop_dag_destroy(self.handle)
        except Exception:
            pass


class Model:
    """predtop_model_create over a host fp32 weight blob (synth.pack_weights order)."""

    def __init__(self, cfg: dict, blob: np.ndarray, device="cuda"):
        self.cfg = ModelConfig(cfg["num_layers"], cfg["d_model"], cfg["num_heads"], cfg["d_ff"],
                               cfg.get("pool", 0), float(cfg.get("ln_eps", 1e-5)))
        nf = lib().predtop_model_weight_floats(ctypes.byref(self.cfg))
        blob = np.ascontiguousarray(blob, np.float32)
        if nf == 0 or nf != blob.size:
            raise PredtopError(UNSUPPORTED if nf == 0 else INVALID_ARG,
                               f"weight blob {blob.size} floats, library expects {nf}")
        nb = lib().predtop_model_device_bytes(ctypes.byref(self.cfg))
        self.device_weights = torch.empty(nb, dtype=torch.uint8, device=device)
        h = ctypes.c_void_p()
        _check(lib().predtop_model_create(ctypes.byref(self.cfg), blob.ctypes.data_as(ctypes.c_void_p),
                                          blob.size, _ptr(self.device_weights), nb, ctypes.byref(h)))
        self.handle = h

    def forward_workspace(self, dag: Dag) -> torch.Tensor:
        n = lib().predtop_stage_forward_workspace(self.handle, dag.handle)
        return torch.empty(n, dtype=torch.uint8, device=self.device_weights.device)

    def forward(self, dag: Dag, workspace: Optional[torch.Tensor] = None, out: Optional[torch.Tensor] = None,
                stream=None) -> torch.Tensor:
        ws = workspace if workspace is not None else self.forward_workspace(dag)
        out = out if out is not None else torch.empty(dag.batch.num_graphs, dtype=torch.float32,
                                                      device=self.device_weights.device)
        predtop_stage_forward(self.handle, dag.handle, ws, out, stream)
        return out

    def node_embeddings(self, dag: Dag, layer: int, workspace: Optional[torch.Tensor] = None,
                        stream=None) -> torch.Tensor:
        ws = workspace if workspace is not None else self.forward_workspace(dag)
        x = torch.empty((dag.batch.total_nodes, self.cfg.d_model), dtype=torch.float32,
                        device=self.device_weights.device)
        _check(lib().predtop_debug_node_embeddings(self.handle, dag.handle, _ptr(ws), ws.numel(), layer,
                                                   _ptr(x), _stream(stream)))
        return x

    def __del__(self):
        try:
            if self.handle and self.handle.value:
                lib().predtop_model_destroy(self.handle)
        except Exception:
            pass


class Plans:
    """Device copy of a synth.PlanSet plus the output / workspace buffers."""

    def __init__(self, plan_ptr, plan_stage, microbatches, device="cuda"):
        self.plan_ptr = torch.as_tensor(np.ascontiguousarray(plan_ptr), dtype=torch.int64).to(device)
        self.plan_stage = torch.as_tensor(np.ascontiguousarray(plan_stage), dtype=torch.int32).to(device)
        self.microbatches = torch.as_tensor(np.ascontiguousarray(microbatches), dtype=torch.int32).to(device)
        self.num_plans = self.plan_ptr.numel() - 1
        self.T = torch.empty(max(self.num_plans, 1), dtype=torch.float64, device=device)
        self.best = torch.empty(1, dtype=torch.int64, device=device)
        self.workspace = torch.empty(int(lib().predtop_plan_latency_workspace()), dtype=torch.uint8, device=device)

    def latency(self, stage_latency: torch.Tensor, no_sync: bool = False, stream=None):
        """Eqn 4 for every plan -> (T tensor, status, first bad plan)."""
        bad = ctypes.c_int64(-1)
        st = lib().predtop_plan_latency(self.num_plans, _ptr(self.plan_ptr), _ptr(self.plan_stage),
                                        _ptr(self.microbatches), _ptr(stage_latency), stage_latency.numel(),
                                        _ptr(self.T), _ptr(self.workspace), self.workspace.numel(),
                                        NO_SYNC if no_sync else 0, ctypes.byref(bad), _stream(stream))
        if st not in (OK, INVALID_ARG):
            _check(st)
        return self.T[:self.num_plans], st, bad.value

    def argmin(self, T: Optional[torch.Tensor] = None, stream=None) -> torch.Tensor:
        T = self.T[:self.num_plans] if T is None else T
        predtop_plan_argmin(T, self.best, stream)
        return self.best


def predtop_plan_search(stage_latency: torch.Tensor, num_layers: int, choice_devices, num_devices: int,
                        microbatches: torch.Tensor, problem_table: Optional[torch.Tensor], T_out, S_out,
                        end_out, choice_out, workspace: torch.Tensor, stream=None):
    """Raw call: stage_latency [num_tables, K, stride] fp32 (device), stage
    (i, j) of choice c at [.., c, tri(i, j)] (include/predtop.h)."""
    nt, K, stride = stage_latency.shape
    assert stage_latency.is_contiguous()
    dev = (ctypes.c_int32 * K)(*[int(x) for x in choice_devices])
    _check(lib().predtop_plan_search(microbatches.numel(), int(num_layers), K, dev, int(num_devices),
                                     _ptr(stage_latency), stride, nt, _ptr(problem_table), _ptr(microbatches),
                                     _ptr(T_out), _ptr(S_out), _ptr(end_out), _ptr(choice_out), _ptr(workspace),
                                     workspace.numel(), _stream(stream)))


def pack_stage_table(dense: np.ndarray) -> np.ndarray:
    """Host helper: dense [L, L, K] (entry (i, j, c), i <= j) -> packed [K, L(L+1)/2]."""
    L, _, K = dense.shape
    iu, ju = np.triu_indices(L)  # row-major upper triangle = tri(i, j) order
    return np.ascontiguousarray(dense[iu, ju, :].T, dtype=np.float32)


class PlanSearch:
    """Inter-stage plan search for P problems over shared
    stage tables: buffers for predtop_plan_search plus host-side decoding."""

    def __init__(self, num_problems: int, num_layers: int, choice_devices, num_devices: int, device="cuda"):
        self.P, self.L = int(num_problems), int(num_layers)
        self.choice_devices = [int(x) for x in choice_devices]
        self.K, self.D = len(self.choice_devices), int(num_devices)
        need = lib().predtop_plan_search_workspace(self.P, self.L, self.K)
        if need == 0:
            raise PredtopError(INVALID_ARG, "plan search sizes out of range")
        self.workspace = torch.empty(need, dtype=torch.uint8, device=device)
        self.T = torch.empty(self.P, dtype=torch.float64, device=device)
        self.S = torch.empty(self.P, dtype=torch.int32, device=device)
        self.ends = torch.zeros((self.P, self.L), dtype=torch.int32, device=device)
        self.choices = torch.zeros((self.P, self.L), dtype=torch.int32, device=device)

    def run(self, stage_latency: torch.Tensor, microbatches: torch.Tensor,
            problem_table: Optional[torch.Tensor] = None, stream=None):
        """stage_latency: [num_tables, K, stride] (pack_stage_table layout)."""
        predtop_plan_search(stage_latency, self.L, self.choice_devices, self.D, microbatches, problem_table,
                            self.T, self.S, self.ends, self.choices, self.workspace, stream)
        return self.T

    def plans(self):
        """Host decode: per problem (T*, [(first, last, choice), ...])."""
        T = self.T.cpu().numpy()
        S = self.S.cpu().numpy()
        E = self.ends.cpu().numpy()
        C = self.choices.cpu().numpy()
        out = []
        for p in range(self.P):
            st, a = [], 0
            for s in range(int(S[p])):
                st.append((a, int(E[p, s]), int(C[p, s])))
                a = int(E[p, s]) + 1
            out.append((float(T[p]), st))
        return out


def prune_graphs(batch: "DeviceBatch", pruned_ops=(OP_RESHAPE, OP_CONVERT_ELEMENT_TYPE), edge_capacity=None,
                 stream=None):
    """predtop_prune_graphs (SIV-B4): raw DeviceBatch -> pruned
    DeviceBatch (device tensors).  Retries once with the exact edge count if
    the first capacity guess (the raw edge count) is too small."""
    dev = batch.node_ptr.device
    desc = batch.desc()
    need = lib().predtop_prune_workspace(ctypes.byref(desc))
    if need == 0:
        raise PredtopError(INVALID_ARG, "invalid batch descriptor")
    ws = torch.empty(need, dtype=torch.uint8, device=dev)
    G = batch.num_graphs
    ops = (ctypes.c_uint16 * len(pruned_ops))(*[int(o) for o in pruned_ops])
    onp = torch.empty(G + 1, dtype=torch.int64, device=dev)
    oep = torch.empty(G + 1, dtype=torch.int64, device=dev)
    ofe = torch.empty(max(batch.total_nodes, 1) * FEAT_BYTES, dtype=torch.uint8, device=dev)
    cap = int(edge_capacity if edge_capacity is not None else max(batch.total_edges, 1))
    tot = (ctypes.c_int64 * 2)()
    bad = ctypes.c_int32(-1)
    for _ in range(2):
        osrc = torch.empty(max(cap, 1), dtype=torch.int32, device=dev)
        odst = torch.empty(max(cap, 1), dtype=torch.int32, device=dev)
        st = lib().predtop_prune_graphs(ctypes.byref(desc), _ptr(batch.node_ptr), _ptr(batch.edge_ptr),
                                        _ptr(batch.src), _ptr(batch.dst), _ptr(batch.feats), ops, len(pruned_ops),
                                        _ptr(ws), ws.numel(), _ptr(onp), _ptr(oep), _ptr(osrc), _ptr(odst), cap,
                                        _ptr(ofe), tot, ctypes.byref(bad), _stream(stream))
        if st == WORKSPACE and tot[1] > cap:
            cap = int(tot[1])
            continue
        _check(st)
        break
    nn, ne = int(tot[0]), int(tot[1])
    sizes = torch.diff(onp).cpu()
    return DeviceBatch(onp, oep, osrc[:ne], odst[:ne], ofe[:nn * FEAT_BYTES],
                       int(sizes.max()) if G else 1)


class Trainer:
    """predtop_train_* over a host fp32 weight blob (synth.pack_weights order):
    fp32 parameters, gradient and Adam moments on the device."""

    PARAMS, GRAD, M, V = 0, 1, 2, 3

    def __init__(self, cfg: dict, blob: np.ndarray, device="cuda"):
        self.cfg = ModelConfig(cfg["num_layers"], cfg["d_model"], cfg["num_heads"], cfg["d_ff"],
                               cfg.get("pool", 0), float(cfg.get("ln_eps", 1e-5)))
        nb = lib().predtop_train_state_bytes(ctypes.byref(self.cfg))
        if nb == 0:
            raise PredtopError(UNSUPPORTED, "unsupported training config")
        blob = np.ascontiguousarray(blob, np.float32)
        self.num_params = blob.size
        self.state = torch.empty(nb, dtype=torch.uint8, device=device)
        h = ctypes.c_void_p()
        _check(lib().predtop_train_create(ctypes.byref(self.cfg), blob.ctypes.data_as(ctypes.c_void_p), blob.size,
                                          _ptr(self.state), nb, ctypes.byref(h)))
        self.handle = h
        self.step = 0
        self._ws = {}

    def buffer(self, which: int) -> torch.Tensor:
        """View of one state blob (PARAMS, GRAD, M, V) as a float32 tensor."""
        p = lib().predtop_train_buffer(self.handle, which)
        off = p - self.state.data_ptr()
        return self.state[off:off + 4 * self.num_params].view(torch.float32)

    def workspace(self, dag: "Dag") -> torch.Tensor:
        n = lib().predtop_train_workspace(self.handle, dag.handle)
        ws = self._ws.get(id(dag))
        if ws is None or ws.numel() < n:
            ws = torch.empty(n, dtype=torch.uint8, device=self.state.device)
            self._ws[id(dag)] = ws
        return ws

    def grad(self, dag: "Dag", y_true: torch.Tensor, stream=None):
        """Forward + MAE loss + backward; returns (loss [1], y_pred [G]) device tensors."""
        ws = self.workspace(dag)
        loss = torch.empty(1, dtype=torch.float32, device=self.state.device)
        y = torch.empty(dag.batch.num_graphs, dtype=torch.float32, device=self.state.device)
        _check(lib().predtop_train_grad(self.handle, dag.handle, _ptr(y_true), _ptr(ws), ws.numel(), _ptr(loss),
                                        _ptr(y), _stream(stream)))
        return loss, y

    def adam(self, lr: float, beta1: float = 0.9, beta2: float = 0.999, eps: float = 1e-8, stream=None):
        self.step += 1
        _check(lib().predtop_train_adam(self.handle, float(lr), self.step, beta1, beta2, eps, _stream(stream)))

    def weights(self) -> np.ndarray:
        """The current fp32 parameters as a host blob."""
        return self.buffer(self.PARAMS).cpu().numpy().copy()

    def __del__(self):
        try:
            if self.handle and self.handle.value:
                lib().predtop_train_destroy(self.handle)
        except Exception:
            pass

