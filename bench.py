#!/usr/bin/env python
"""bench.py -- PredTOP prediction path on B200.

One step = the whole hot path over one batch: predtop_build_dag (validate,
depth, closure, mask) + predtop_stage_forward (DAG-Transformer, 4 layers) +
predtop_plan_latency (Eqn 4) + [N>1: NCCL all-gather of plan latencies] +
predtop_plan_argmin.  Default workload per GPU (the largest single-GPU config,
BASELINE.json configs[2]): 512 MoE-style stage DAGs of 1350-1650 ops (seeded,
synthetic), d=256, 8 heads, d_ff=1024; 128 plans of 4 stages x 16 microbatches
(owned mode); configs[1] (1024 GPT-style DAGs, d=128) is measured in the same
run and reported under "also".  Weak scaling: rank r scores graphs
[G r, G (r+1)).  `--gpus N` without a torchrun environment re-launches itself
under torch.distributed.run with N ranks.

Timing: W warm-up steps, then K steps, each preceded by an untimed L2 flush
(256 MiB memset > 126 MB L2) and bracketed by CUDA events on the compute
stream; barrier + synchronize around the timed region; max over ranks.
`value` = graphs scored per second over all ranks.  `e2e` repeats the step
through the same C-ABI with pinned HOST inputs (H2D inside the timed region)
and reads the plan latencies back (D2H).  A second, separate pass with
predtop_profile_enable times every kernel with CUDA events on its launch
stream; the dominant kernel gives the `roofline` object.

--impl reference times the CPU fp64 oracle (oracle/, test infrastructure) on
a bounded sample of the same workload on the host cores.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "candidate stage-DAGs scored/sec"
UNIT = "graphs/s"
PEAKS_FALLBACK = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0,
                  "sm_max_mhz": 1965.0}
MUFU_EX2_PER_CLK_SM = 16  # sm_100 SFU ex2 rate per SM per clock
NUM_SMS = 148


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d, "measured"
    return PEAKS_FALLBACK, "fallback"


# ----------------------------------------------------------------- clocks
class ClockSampler:
    """Samples SM clock and clock-event reasons with NVML during the timed region."""
    REASONS = {0x2: "applications_clocks", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown"}

    def __init__(self, device_index: int):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        self._t = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        nv = self.nv
        get_reasons = getattr(nv, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
            getattr(nv, "nvmlDeviceGetCurrentClocksThrottleReasons")
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = get_reasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.01)

    def __enter__(self):
        if self.nv:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        return {"sm_mhz": float(statistics.median(self.samples)) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                "samples": len(self.samples)}


# ----------------------------------------------------------------- oracle leg
def host_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def oracle_rate(cfg, blob, batch, target_s: float = 15.0, max_graphs: int = 1024, hops: int = 0):
    """Oracle graphs/s on a bounded sample (the first n graphs) with all host
    cores; also returns the oracle latencies of the sample (parity)."""
    import oracle
    oracle.build()
    cores = host_cores()
    t0 = time.perf_counter()
    oracle.forward_batch(cfg, blob, batch, graphs=[0], threads=1, hops=hops)
    t1 = time.perf_counter() - t0
    n = int(max(cores, min(max_graphs, batch.num_graphs, round(target_s * cores / max(t1, 1e-6)))))
    n = min(n, batch.num_graphs)
    t0 = time.perf_counter()
    y = oracle.forward_batch(cfg, blob, batch, graphs=list(range(n)), threads=cores, hops=hops)
    wall = time.perf_counter() - t0
    return n / wall, cores, n, wall, y


def parity_stats(y_gpu, y_oracle, cond=None):
    """GPU-vs-oracle relative error per graph (north star: <= 2e-3); with
    `cond` (oracle.head_condition of the first len(cond) graphs) also the
    bias-free error |dy| / sum_i |w_o,i h2_i| (R17, R22)."""
    y = np.asarray(y_gpu, np.float64)
    w = np.asarray(y_oracle, np.float64)
    r = np.abs(y - w) / np.abs(w)
    out = {"max_rel": float(r.max()), "median_rel": float(np.median(r)), "graphs": int(len(y)),
           "tolerance": 2e-3, "pass": bool(r.max() <= 2e-3)}
    if cond is not None and len(cond):
        c = np.asarray(cond, np.float64)
        rb = np.abs(y[:len(c)] - w[:len(c)]) / c
        out.update({"max_rel_nobias": float(rb.max()), "median_rel_nobias": float(np.median(rb)),
                    "graphs_nobias": int(len(c)), "pass": bool(r.max() <= 2e-3 and rb.max() <= 2e-3)})
    return out


def run_reference(args, rank):
    if rank != 0:
        return
    if args.config == "16k":
        return run_reference_16k(args)
    from paper_conf_ipps_acharyas25_b200 import synth
    import oracle
    oracle.build()
    if args.config == "train":  # the oracle's fp64 MAE gradient (orc_grad) + Adam on mini-batches
        cfg = dict(synth.MODEL_CONFIGS["paper"])
        blob = synth.pack_weights(cfg, synth.model_weights(cfg)).astype(np.float64)
        cores = host_cores()
        nb = cores
        batch = synth.stage_batch("gpt", nb)
        yl = 0.01 * np.diff(batch.node_ptr) + 1.0
        m, v = np.zeros_like(blob), np.zeros_like(blob)
        t_total = 0.0
        for s_ in range(min(args.warmup, 1) + args.steps):
            t0 = time.perf_counter()
            _, g, _ = oracle.mae_grad(cfg, blob.astype(np.float32), batch, yl, threads=cores)
            blob, m, v = oracle.adam_step(blob, g, m, v, s_ + 1, 1e-3)
            if s_ >= min(args.warmup, 1):
                t_total += time.perf_counter() - t0
        value = nb * args.steps / t_total
        line = {"impl": "reference", "metric": "stage-DAGs trained/sec (forward + MAE + backward + Adam)",
                "value": value, "unit": "graphs/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": 1000 * t_total / args.steps, "higher_is_better": True, "scaling": "weak",
                "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": f"train: mini-batches of {nb} GPT-style stage DAGs, paper model (P:178)"},
                "cpu_baseline": {"value": value, "unit": "graphs/s", "cores": cores, "kind": "oracle",
                                 "sample": f"{args.steps} steps x {nb} graphs, fp64 orc_grad + Adam"},
                "e2e": {"value": value, "unit": "graphs/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line), flush=True)
        return
    gcfg = "gpt" if args.config in ("sweep", "search") else args.config  # sweep stages are GPT-style pool graphs
    cfg = synth.MODEL_CONFIGS[gcfg]
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    cores = host_cores()
    per_step = cores  # one graph per core per step
    nb = min(per_step * (min(args.warmup, 1) + args.steps), 4096 if gcfg == "gpt" else 512)
    batch = synth.tiny_batch() if gcfg == "tiny" else synth.stage_batch(gcfg, nb)
    plans_B = plan_microbatches(args.config)
    done, t_total = 0, 0.0
    # a CPU program has nothing to warm beyond its first step: one untimed
    # warm-up step whatever W is (an MoE step is ~5-10 s of oracle work)
    nwarm = min(args.warmup, 1)
    for s in range(nwarm + args.steps):
        gs = [(s * per_step + i) % batch.num_graphs for i in range(per_step)]
        t0 = time.perf_counter()
        y = oracle.forward_batch(cfg, blob, batch, graphs=gs, threads=cores)
        # plan formula over the sampled stages (owned mode, 4 stages x B = 16)
        S = stages_per_plan(args.config, len(gs))
        P = len(gs) // S
        if P:
            oracle.plan_T(np.arange(P + 1) * S, np.arange(S * P), np.full(P, plans_B), y[:S * P].astype(np.float32))
        dt = time.perf_counter() - t0
        if s >= nwarm:
            done += len(gs)
            t_total += dt
    value = done / t_total
    sample = f"{args.steps} steps x {per_step} {args.config} stage graphs (one per host core), fp64 oracle"
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * t_total / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": workload_config(args),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


CONFIG_TEXT = {
    "tiny": "4 hand-made DAGs of 8-16 ops (chain, diamond, fan-out, chain with skips), 1 layer d=32 H=2 d_ff=128",
    "gpt": "stage DAGs of 270-330 ops (fwd+bwd GPT-3 1.3B stage template), 4 layers d=128 H=8 d_ff=512",
    "moe": "stage DAGs of 1350-1650 ops (fwd+bwd GShard-MoE 2.6B stage template, 16-expert fan-out), "
           "4 layers d=256 H=8 d_ff=1024",
    "16k": "stage DAGs of exactly 16384 ops (GPT-style template), 4 layers d=128 H=8 d_ff=512",
}


def stages_per_plan(config: str, G: int) -> int:
    """tiny: 1-stage plans (BASELINE configs[0]); else 4-stage plans."""
    return 1 if config == "tiny" else max(1, min(4, G))


def plan_microbatches(config: str) -> int:
    return 4 if config == "tiny" else 16


def run_reference_16k(args):
    """--impl reference for configs[3]: the oracle on the 16 384-op DAG, its
    layers evaluated row block by row block on all host cores
    (oracle.forward_rows); one step = one whole forward (~30-60 s), so the
    run times min(steps, 1) step after no warm-up."""
    from paper_conf_ipps_acharyas25_b200 import synth
    import oracle
    oracle.build()
    cfg = synth.MODEL_CONFIGS["16k"]
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    cores = host_cores()
    b = synth.stage_batch("16k", 1)
    tm = {}
    oracle.forward_rows(cfg, blob, *b.graph(0), threads=cores, timings=tm)
    value = 1.0 / tm["total_s"]
    sample = (f"1 whole 16k stage graph (depth, closure, mask single-threaded {tm['graph_steps_s']:.1f} s; "
              f"4 layers row-parallel on {cores} threads {sum(tm['layers_s']):.1f} s), fp64 oracle")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": 1, "warmup": 0, "ms_per_step": 1000 * tm["total_s"], "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": workload_config(args),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def workload_config(args):
    cfg_name = "gpt" if args.config in ("sweep", "search") else args.config
    from paper_conf_ipps_acharyas25_b200 import synth
    c = synth.MODEL_CONFIGS[cfg_name]
    base = {"layers": c["num_layers"], "d_model": c["d_model"], "heads": c["num_heads"], "d_ff": c["d_ff"],
            "precision": "f16 MMA operands, f32 accumulate/softmax/LN/residual, f32 latency, f64 Eqn 4"}
    if args.config == "sweep":
        return dict({"workload": f"sweep: {args.plans} candidate plans (S~U{{2..8}} stages, B~U{{1,4,16,64}}), "
                                 f"each owning its GPT-style stage graphs ({CONFIG_TEXT['gpt']}), scored in chunks "
                                 f"of {args.chunk} graphs; Eqn 4 per plan; global argmin",
                     "plans_total": args.plans, "chunk_graphs": args.chunk, "stage_pool": args.pool,
                     "parallelism": f"plan-sharded x{args.gpus} (cost-balanced contiguous ranges), "
                                    f"NCCL all-gather of plan latencies",
                     "l2": "inputs and activations of one step (~500k graphs) far exceed the 126 MB L2"}, **base)
    G, S, B = args.graphs, stages_per_plan(args.config, args.graphs), plan_microbatches(args.config)
    return dict({"workload": f"{args.config}: {G} {CONFIG_TEXT[args.config]}, sum pool + MLP head; "
                             f"{G // S} plans x {S} stages x B={B} (Eqn 4)",
                 "graphs_per_gpu": G, "plans_per_gpu": G // S, "stages_per_plan": S, "microbatches": B,
                 "parallelism": f"graph-sharded x{args.gpus} (owned plans), NCCL all-gather of plan latencies",
                 "l2": "flushed before every timed step (256 MiB memset, untimed)",
                 "dagra_k": args.hops if args.hops > 0 else "inf"}, **base)


# ----------------------------------------------------------------- main leg
DEFAULT_GRAPHS = {"tiny": 4, "gpt": 1024, "moe": 512, "16k": 1, "sweep": 0, "search": 0, "train": 32}
ALSO_KEYS = ("metric", "value", "unit", "ms_per_step", "steps", "config", "e2e", "gpu_launches", "roofline",
             "cpu_baseline", "parity", "result", "clocks")


class Ctx:
    """Per-rank run context: device, stream, process group, timing helpers."""

    def __init__(self, args):
        import torch
        import torch.distributed as dist
        self.torch, self.dist = torch, dist
        self.rank = int(os.environ.get("RANK", "0"))
        self.world = int(os.environ.get("WORLD_SIZE", "1"))
        local = int(os.environ.get("LOCAL_RANK", "0"))
        self.gloo = args.dist_backend == "gloo"
        if self.gloo:
            args.eager = True  # a host-side collective cannot sit inside a CUDA graph
        self.dev_index = local % torch.cuda.device_count() if self.gloo else local
        torch.cuda.set_device(self.dev_index)
        self.dev = torch.device("cuda", self.dev_index)
        if self.world > 1:
            if self.gloo:
                dist.init_process_group("gloo")
            else:
                dist.init_process_group("nccl", device_id=self.dev)
        from paper_conf_ipps_acharyas25_b200 import build
        if self.rank == 0:
            build.build_library()
        if self.world > 1:
            dist.barrier()
        from paper_conf_ipps_acharyas25_b200 import predtop as pt
        self.pt = pt
        self.L = pt.lib()
        self.stream = torch.cuda.current_stream()
        self.flush = torch.empty(256 << 20, dtype=torch.uint8, device=self.dev)

    def timed(self, fn, k, flush=True):
        torch, dist = self.torch, self.dist
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(k)]
        if self.world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        for a, b in evs:
            if flush:
                self.flush.zero_()
            a.record(self.stream)
            fn()
            b.record(self.stream)
        torch.cuda.synchronize()
        if self.world > 1:
            dist.barrier()
        return [a.elapsed_time(b) for a, b in evs]

    def max_over_ranks(self, x):
        if self.world > 1:
            t = self.torch.tensor([x], dtype=self.torch.float64, device="cpu" if self.gloo else self.dev)
            self.dist.all_reduce(t, op=self.dist.ReduceOp.MAX)
            return float(t.item())
        return x

    def sum_over_ranks(self, x):
        if self.world > 1:
            t = self.torch.tensor([x], dtype=self.torch.float64, device="cpu" if self.gloo else self.dev)
            self.dist.all_reduce(t, op=self.dist.ReduceOp.SUM)
            return float(t.item())
        return x

    def all_gather_T(self, T_all, T):
        if self.gloo:
            P = T.numel()
            parts = [self.torch.empty(P, dtype=self.torch.float64) for _ in range(self.world)]
            self.dist.all_gather(parts, T.cpu())
            T_all.copy_(self.torch.cat(parts))
        else:
            self.dist.all_gather_into_tensor(T_all, T)

    def capture(self, fn):
        """CUDA-graph capture of fn (library calls are capturable: NO_SYNC
        build, stream-ordered kernels, NCCL all-gather); returns (replay, launches)."""
        torch = self.torch
        side = torch.cuda.Stream(device=self.dev)
        side.wait_stream(self.stream)
        with torch.cuda.stream(side):
            fn()
        self.stream.wait_stream(side)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        l0 = self.L.predtop_launch_count()
        try:
            with torch.cuda.graph(g, stream=side):
                fn()
        except RuntimeError as e:  # e.g. a collective backend that cannot be captured: run eagerly
            print(f"bench: CUDA-graph capture failed ({e}); timing eager steps", file=sys.stderr)
            torch.cuda.synchronize()
            self.capture_failed = True
            return fn, None
        n = self.L.predtop_launch_count() - l0
        torch.cuda.synchronize()
        self._graphs = getattr(self, "_graphs", []) + [g]
        return g.replay, n

    def profile(self, step, steps):
        """Per-kernel CUDA-event times (predtop_profile_enable) over `steps` eager steps."""
        import ctypes
        L = self.L
        L.predtop_profile_enable(1)
        self.timed(step, steps)
        L.predtop_profile_enable(0)
        kinds = 32
        kms = (ctypes.c_double * kinds)()
        kcnt = (ctypes.c_int64 * kinds)()
        nk = L.predtop_profile_read(kms, kcnt, kinds)
        names = [L.predtop_profile_kind_name(i).decode() for i in range(nk)]
        return {names[i]: {"ms_per_step": kms[i] / steps, "launches_per_step": kcnt[i] / steps}
                for i in range(nk) if kcnt[i]}

    def finish(self):
        if self.world > 1:
            self.dist.barrier()
            self.dist.destroy_process_group()


def algorithmic_work(cfg, node_total, edge_total, words, pairs):
    """Algorithmic work per step of each kernel kind: flops for
    tensor-bound kinds, exps for the attention (MUFU-bound), bytes for HBM-bound."""
    d, dff, H = cfg["d_model"], cfg["d_ff"], cfg["num_heads"]
    N, E, A = float(node_total), float(edge_total), float(pairs)
    return {
        "gemm_qkv": ("tensor", 2.0 * N * d * 3 * d),
        "gemm_oproj_ln": ("tensor", 2.0 * N * d * d),
        "gemm_ffn1": ("tensor", 2.0 * N * d * dff),
        "gemm_ffn2_ln": ("tensor", 2.0 * N * dff * d),
        "layer_tail": ("tensor", 2.0 * N * (d * d + 2 * d * dff)),
        "attention": ("alu", float(H) * A),  # exps per layer (MUFU-bound)
        "dag_closure": ("hbm", 8.0 * words + 8.0 * E),
        "dag_mask": ("hbm", 3 * 8.0 * words),
        "readout": ("hbm", 4.0 * N * d),
        "embed": ("hbm", N * (20.0 + 4 + 6 * d)),
    }


def roofline(prof, work, cfg, pairs, node_total, clk, step_ms):
    """The dominant kernel's achieved rate against its peak.  `work` is per STEP;
    per launch = per step / launches per step; time per launch from the
    CUDA-event profile pass."""
    for k in prof:
        prof[k]["share"] = prof[k]["ms_per_step"] / step_ms
    peaks, peak_src = load_peaks()
    dom = max(prof, key=lambda k: prof[k]["ms_per_step"]) if prof else None
    if dom not in work:
        return None
    bound, per_step = work[dom]
    n_l = prof[dom]["launches_per_step"]
    per_launch_ms = prof[dom]["ms_per_step"] / n_l
    layer_kinds = ("gemm_qkv", "gemm_oproj_ln", "gemm_ffn1", "gemm_ffn2_ln", "layer_tail", "attention")
    # work[] holds per-layer figures for the per-layer kernels, per-step figures otherwise
    units = (per_step * cfg["num_layers"] if dom in layer_kinds else per_step) / n_l
    sec = per_launch_ms / 1e3
    d = cfg["d_model"]
    if bound == "tensor":
        ach = units / sec / 1e12
        peak, basis = tensor_peak(peaks, clk)
        roof = {"bound": "tensor", "achieved": ach, "peak": peak, "unit": "TFLOP/s", "frac": ach / peak,
                "peak_basis": basis + "; f16 MMA has the same nominal rate"}
    elif bound == "hbm":
        ach = units / sec / 1e9
        roof = {"bound": "hbm", "achieved": ach, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": ach / peaks["hbm_gbs"]}
    else:
        clk_mhz = (clk.summary()["sm_mhz"] or peaks.get("sm_max_mhz", 1965.0))
        peak = MUFU_EX2_PER_CLK_SM * NUM_SMS * clk_mhz * 1e6 / 1e9
        ach = units / sec / 1e9
        A_launch = float(pairs) * cfg["num_layers"] / n_l
        tflops = 4.0 * d * A_launch / sec / 1e12
        roof = {"bound": "alu", "achieved": ach, "peak": peak, "unit": "Gexp/s", "frac": ach / peak,
                "peak_basis": f"MUFU ex2 {MUFU_EX2_PER_CLK_SM}/clk/SM x {NUM_SMS} SMs x {clk_mhz:.0f} MHz "
                              f"(median under load)",
                "tensor_equiv_tflops": tflops,
                "tensor_frac": tflops / tensor_peak(peaks, clk)[0]}
    traffic = None
    try:  # DRAM bytes per launch of the dominant kernel from a committed ncu capture
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            tdb = json.load(f)
        name = cfg.get("_name", "gpt")
        tr = tdb.get(f"{name}/{dom}") or tdb.get(dom)
        if tr and tr.get("config", "gpt") == name:
            traffic = tr["bytes"]
            roof["traffic_source"] = tr["source"]
            if dom == "attention":  # algorithmic bytes: q,k,v in (3d fp16) + att out (d fp16) per node
                roof["traffic_algorithmic"] = float(node_total) * 4 * d * 2 * cfg["num_layers"] / n_l
    except (OSError, ValueError, KeyError):
        traffic = None
    roof.update({"kernel": dom, "traffic": traffic, "peak_source": peak_src,
                 "kernel_ms": per_launch_ms, "share_of_step": prof[dom]["share"]})
    return roof


def tensor_peak(peaks, clk):
    """The dense f16/bf16 tensor peak that applies to this run: the measured
    burst figure when the SM clock under load stayed near its maximum (the
    sustained figure is a 4 s back-to-back cuBLAS run that power-throttles
    to ~1.3 GHz; this step's kernels do not), else the sustained one."""
    smax = peaks.get("sm_max_mhz", 1965.0)
    med = clk.summary()["sm_mhz"] if clk is not None else None
    if med and med >= 0.9 * smax:
        return peaks["bf16_tflops"], f"measured cuBLAS bf16 burst (SM clock under load {med:.0f} of {smax:.0f} MHz)"
    return (peaks.get("bf16_tflops_sustained", peaks["bf16_tflops"]),
            f"measured cuBLAS bf16 sustained (SM clock under load {med} MHz)")


def kernel_rooflines(prof, cfg, node_total, edge_total, words, pairs, clk):
    """Every kernel's algorithmic work / its measured time against its own
    bound, plus the layer stack (projections + attention + FFN)
    as one tensor-roofline fraction.  Per step; per-layer kinds x num_layers."""
    peaks, _ = load_peaks()
    tpk, tbasis = tensor_peak(peaks, clk)
    hbm = peaks["hbm_gbs"]
    d, dff, H, Lm = cfg["d_model"], cfg["d_ff"], cfg["num_heads"], cfg["num_layers"]
    N, E, A = float(node_total), float(edge_total), float(pairs)
    clk_mhz = clk.summary()["sm_mhz"] or peaks.get("sm_max_mhz", 1965.0)
    mufu = MUFU_EX2_PER_CLK_SM * NUM_SMS * clk_mhz * 1e6
    out = {}

    def sec(k):
        return prof[k]["ms_per_step"] / 1e3 if k in prof else None

    def put(k, bound, work, peak, unit):
        t = sec(k)
        if t:
            ach = work / t
            out[k] = {"bound": bound, "achieved": ach / (1e12 if unit == "TFLOP/s" else 1e9),
                      "peak": peak, "unit": unit, "frac": ach / (peak * (1e12 if unit == "TFLOP/s" else 1e9))}

    put("gemm_qkv", "hbm", Lm * N * (2 * d + 6 * d), hbm, "GB/s")
    put("attention", "alu", Lm * H * A, mufu / 1e9, "Gexp/s")
    put("layer_tail", "tensor", Lm * 2 * N * (d * d + 2 * d * dff), tpk, "TFLOP/s")
    put("embed", "hbm", N * (20.0 + 4 + 6 * d), hbm, "GB/s")
    put("readout", "hbm", 4.0 * N * d, hbm, "GB/s")
    put("dag_small", "hbm", 8.0 * E + 4.0 * N + 2 * 8.0 * words, hbm, "GB/s")
    t_layers = sum(sec(k) or 0.0 for k in ("gemm_qkv", "attention", "layer_tail", "gemm_oproj_ln", "gemm_ffn1",
                                             "gemm_ffn2_ln"))
    if t_layers:
        fl = Lm * (2 * N * (3 * d * d + d * d + 2 * d * dff) + 4.0 * d * A)
        out["layer_stack"] = {"bound": "tensor", "achieved": fl / t_layers / 1e12, "peak": tpk, "unit": "TFLOP/s",
                              "frac": fl / t_layers / 1e12 / tpk,
                              "note": "QKV + attention (4 d |A|) + O-proj + FFN flops over the time of those kernels"}
    out["tensor_peak_basis"] = tbasis
    return out


def dag_pairs(pt, dag, sizes):
    T_ = (np.asarray(sizes) + 127) // 128
    _, pairs = dag.tiles(int((T_ * T_).sum()))
    return int(pairs.sum().item())


def run_batch(args, ctx):
    """configs tiny/gpt/moe/16k: one step = build + forward of the rank's G graphs,
    Eqn 4 over its owned plans, all-gather, global argmin."""
    import torch
    from paper_conf_ipps_acharyas25_b200 import synth
    pt, L, dev, world, rank = ctx.pt, ctx.L, ctx.dev, ctx.world, ctx.rank

    cfg = dict(synth.MODEL_CONFIGS[args.config], _name=args.config)
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    G = args.graphs
    host = synth.tiny_batch() if args.config == "tiny" else synth.stage_batch(args.config, G, first_graph=rank * G)
    S = stages_per_plan(args.config, G)
    ps = synth.owned_plans(G, S, plan_microbatches(args.config))
    model = pt.Model(cfg, blob, device=dev)
    db = pt.DeviceBatch.from_host(host, device=dev)
    dag = pt.Dag(db, no_sync=True, hops=args.hops)
    ws = model.forward_workspace(dag)
    lat = torch.empty(G, dtype=torch.float32, device=dev)
    plans = pt.Plans(ps.plan_ptr, ps.plan_stage, ps.microbatches, device=dev)
    P = plans.num_plans
    T_all = torch.empty(world * P, dtype=torch.float64, device=dev)

    def step():
        dag.rebuild()                       # predtop_build_dag (NO_SYNC)
        model.forward(dag, ws, lat)         # predtop_stage_forward
        T, _, _ = plans.latency(lat, no_sync=True)   # predtop_plan_latency
        if world > 1:
            ctx.all_gather_T(T_all, T)
            plans.argmin(T_all)             # global argmin by (T, global plan id)
        else:
            plans.argmin(T)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    st, bad = dag.dag_status()
    assert st == pt.OK, (st, bad)
    assert torch.isfinite(lat).all()

    # eager diagnostics: host enqueue time of one step and eager device time
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(5):
        step()
    host_enqueue_ms = (time.perf_counter() - t0) / 5 * 1e3
    torch.cuda.synchronize()
    eager_ms = sum(ctx.timed(step, 5)) / 5

    launches_per_step = None
    if not args.eager:
        run, launches_per_step = ctx.capture(step)
    else:
        run = step
    run()
    torch.cuda.synchronize()

    launches0 = L.predtop_launch_count()
    with ClockSampler(ctx.dev_index) as clk:
        ms = ctx.timed(run, args.steps)
    launches = L.predtop_launch_count() - launches0
    if launches_per_step is not None:
        launches = launches_per_step * args.steps
    total_ms = ctx.max_over_ranks(sum(ms))
    value = world * G * args.steps / (total_ms / 1e3)
    plans_per_s = world * P * args.steps / (total_ms / 1e3)
    assert torch.isfinite(lat).all()
    # the plan latencies of ALL ranks (gathered) and the global best plan: a
    # 1-rank run over world*G graphs gives bitwise the same (tests/test_bench_ranks.py)
    import hashlib
    T_fin = (T_all if world > 1 else plans.T[:P]).cpu().numpy()
    result = {"T_sha256": hashlib.sha256(T_fin.tobytes()).hexdigest(), "plans": int(T_fin.size),
              "best_plan": int(plans.best.item()) if P else None}
    if args.no_extras:
        if rank == 0:
            emit({"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                  "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
                  "scaling": "weak", "vs_baseline": None, "dtype": "f16", "data": "synthetic",
                  "config": workload_config(args), "plans_per_s": plans_per_s, "result": result,
                  "launch_mode": "eager" if args.eager or getattr(ctx, "capture_failed", False) else "cuda_graph",
                  "clocks": clk.summary(), "note": "--no-extras: e2e, profile, cpu_baseline skipped"}, args)
        return

    # ---- e2e through the C-ABI with pinned host buffers
    pin = {
        "node_ptr": torch.from_numpy(host.node_ptr).pin_memory(),
        "edge_ptr": torch.from_numpy(host.edge_ptr).pin_memory(),
        "src": torch.from_numpy(host.src).pin_memory(),
        "dst": torch.from_numpy(host.dst).pin_memory(),
        "feats": torch.from_numpy(np.ascontiguousarray(host.feats).view(np.uint8).reshape(-1).copy()).pin_memory(),
        "plan_ptr": torch.from_numpy(ps.plan_ptr).pin_memory(),
        "plan_stage": torch.from_numpy(ps.plan_stage).pin_memory(),
        "mb": torch.from_numpy(ps.microbatches).pin_memory(),
    }
    T_host = torch.empty(max(world * P, 1), dtype=torch.float64).pin_memory()
    best_host = torch.empty(1, dtype=torch.int64).pin_memory()
    h2d = sum(t.numel() * t.element_size() for t in pin.values())
    d2h = world * P * 8 + 8

    def e2e_step():
        db.node_ptr.copy_(pin["node_ptr"], non_blocking=True)
        db.edge_ptr.copy_(pin["edge_ptr"], non_blocking=True)
        db.src.copy_(pin["src"], non_blocking=True)
        db.dst.copy_(pin["dst"], non_blocking=True)
        db.feats.copy_(pin["feats"], non_blocking=True)
        plans.plan_ptr.copy_(pin["plan_ptr"], non_blocking=True)
        plans.plan_stage.copy_(pin["plan_stage"], non_blocking=True)
        plans.microbatches.copy_(pin["mb"], non_blocking=True)
        step()
        if P:
            T_host[:world * P].copy_(T_all if world > 1 else plans.T[:P], non_blocking=True)
        best_host.copy_(plans.best, non_blocking=True)

    e2e_run = e2e_step if args.eager else ctx.capture(e2e_step)[0]
    for _ in range(2):
        e2e_run()
    ms_e2e = ctx.timed(e2e_run, max(10, args.steps // 4))
    tot_e2e = ctx.max_over_ranks(sum(ms_e2e))
    e2e_serial = world * G * len(ms_e2e) / (tot_e2e / 1e3)
    torch.cuda.synchronize()
    if P:  # the host copy of the plan latencies matches the device result
        assert torch.equal(T_host[:world * P], (T_all if world > 1 else plans.T[:P]).cpu())

    # ---- e2e pipelined: two input buffer sets; the host->device copy of step
    # i+1 runs on a copy stream while step i computes (each step still copies
    # its own inputs inside the timed region and reads its result back)
    e2e_value, e2e_mode = e2e_serial, "serial"
    if not args.eager and world == 1:
        db2 = pt.DeviceBatch(db.node_ptr.clone(), db.edge_ptr.clone(), db.src.clone(), db.dst.clone(),
                             db.feats.clone(), db.max_nodes)
        dag2 = pt.Dag(db2, no_sync=True, hops=args.hops)
        plans2 = pt.Plans(ps.plan_ptr, ps.plan_stage, ps.microbatches, device=dev)
        sets = [(db, dag, plans), (db2, dag2, plans2)]

        def make_step(k):
            dbk, dagk, plk = sets[k]

            def f():
                dagk.rebuild()
                model.forward(dagk, ws, lat)
                T, _, _ = plk.latency(lat, no_sync=True)
                plk.argmin(T)
                if P:
                    T_host[:P].copy_(plk.T[:P], non_blocking=True)
                best_host.copy_(plk.best, non_blocking=True)
            return f

        graphs = [ctx.capture(make_step(k))[0] for k in range(2)]
        cs = torch.cuda.Stream(device=dev)
        ev_in = [torch.cuda.Event(), torch.cuda.Event()]
        ev_done = [torch.cuda.Event(), torch.cuda.Event()]

        def copy_in(k):
            dbk, _, plk = sets[k]
            with torch.cuda.stream(cs):
                cs.wait_event(ev_done[k])  # step k-2 finished with buffer set k
                dbk.node_ptr.copy_(pin["node_ptr"], non_blocking=True)
                dbk.edge_ptr.copy_(pin["edge_ptr"], non_blocking=True)
                dbk.src.copy_(pin["src"], non_blocking=True)
                dbk.dst.copy_(pin["dst"], non_blocking=True)
                dbk.feats.copy_(pin["feats"], non_blocking=True)
                plk.plan_ptr.copy_(pin["plan_ptr"], non_blocking=True)
                plk.plan_stage.copy_(pin["plan_stage"], non_blocking=True)
                plk.microbatches.copy_(pin["mb"], non_blocking=True)
                ev_in[k].record(cs)

        def pipelined(n):
            copy_in(0)
            for i in range(n):
                k = i & 1
                if i + 1 < n:
                    copy_in(k ^ 1)
                ctx.stream.wait_event(ev_in[k])
                graphs[k]()
                ev_done[k].record(ctx.stream)

        pipelined(4)
        torch.cuda.synchronize()
        n_e2e = max(10, args.steps)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record(ctx.stream)
        pipelined(n_e2e)
        b.record(ctx.stream)
        torch.cuda.synchronize()
        e2e_value = G * n_e2e / (a.elapsed_time(b) / 1e3)
        e2e_mode = (f"pipelined: {n_e2e} steps back to back, the H2D copy of step i+1 (copy stream) "
                    f"overlaps step i; every step copies its inputs and reads T* back; no L2 flush")
        if P:
            assert torch.equal(T_host[:P], plans.T[:P].cpu())

    # ---- per-kernel profile pass (separate from the headline timing)
    prof = ctx.profile(step, max(5, args.steps // 4))
    words = int(sum(n * 2 * ((n + 127) // 128) for n in host.sizes))
    A = dag_pairs(pt, dag, host.sizes)
    work = algorithmic_work(cfg, host.node_ptr[-1], host.edge_ptr[-1], words, A)
    roof = roofline(prof, work, cfg, A, host.node_ptr[-1], clk, total_ms / args.steps)
    kroof = kernel_rooflines(prof, cfg, host.node_ptr[-1], host.edge_ptr[-1], words, A, clk)

    cpu, parity = None, None
    y_gpu = lat.cpu().numpy().astype(np.float64)
    if rank == 0 and world == 1 and not args.no_cpu_baseline and args.config == "16k":
        import oracle
        oracle.build()
        cores = host_cores()
        tm = {}
        _, y16, _ = oracle.forward_rows(cfg, blob, *host.graph(0), threads=cores, timings=tm)
        cpu = {"value": 1.0 / tm["total_s"], "unit": UNIT, "cores": cores, "kind": "oracle",
               "sample": f"the whole 16k stage graph: depth, closure, mask {tm['graph_steps_s']:.1f} s "
                         f"(single-threaded) + 4 layers {sum(tm['layers_s']):.1f} s (row blocks on {cores} threads), "
                         f"fp64 C oracle"}
        parity = parity_stats(y_gpu[:1], [y16])
    elif rank == 0 and world == 1 and not args.no_cpu_baseline:
        v, cores, n, wall, y_or = oracle_rate(cfg, blob, host, hops=getattr(args, "hops", 0))
        cpu = {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle",
               "sample": f"first {n} of {G} {args.config} stage graphs, fp64 C oracle, {cores} threads, {wall:.1f} s"}
        import oracle
        m = min(n, 16)
        _, cond = oracle.forward_batch_cond(cfg, blob, host, graphs=list(range(m)), threads=cores,
                                            hops=getattr(args, "hops", 0))
        parity = parity_stats(y_gpu[:n], y_or, cond)
        parity["sample"] = f"the {n} cpu_baseline graphs"

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "f16", "data": "synthetic",
                "config": workload_config(args),
                "plans_per_s": plans_per_s,
                "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
                        "d2h_bytes_per_step": int(d2h), "mode": e2e_mode, "serial_value": e2e_serial},
                "gpu_launches": int(launches),
                "launch_mode": "eager" if args.eager or getattr(ctx, "capture_failed", False) else "cuda_graph",
                "eager_ms_per_step": eager_ms, "host_enqueue_ms_per_step": host_enqueue_ms,
                "roofline": roof, "kernel_rooflines": kroof, "cpu_baseline": cpu, "parity": parity,
                "result": result, "clocks": clk.summary(),
                "kernels": {k: {kk: round(vv, 5) for kk, vv in v.items()} for k, v in prof.items()}}
        return line
    return None


def run_search(args, ctx):
    """the shared stage table + plan search.  All L(L+1)/2
    layer-range stages of GPT-3 1.3B (24 layers, Table IV) scored by one
    model per Table III mesh choice (6), stage DAGs cost-balanced over the
    ranks, one exact sum-all-reduce of the stage table, then the plan search
    on Platform 2's 4 GPUs for B in {1..64} (7 problems)."""
    import torch
    from paper_conf_ipps_acharyas25_b200 import synth, stage_table
    pt, L, dev, world, rank = ctx.pt, ctx.L, ctx.dev, ctx.world, ctx.rank
    nl = args.layers
    host = synth.layer_range_stages("gpt", nl)
    cfgs = synth.mesh_model_configs("search", len(synth.MESH_CHOICES))
    blobs = [synth.pack_weights(c, synth.model_weights(c)) for c in cfgs]
    devs = [d for _, d in synth.MESH_CHOICES]
    Bs = [1, 2, 4, 8, 16, 32, 64]
    sts = stage_table.StageTableSearch(pt, cfgs, blobs, host, nl, devs, 4, Bs, rank=rank, world=world,
                                       device=dev, hops=args.hops)
    K, NT = len(cfgs), sts.NT
    step = sts.step
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    tab = sts.table.cpu().numpy()
    assert np.isfinite(tab).all() and (tab > 0).all(), "stage latencies must be positive (R17)"
    run, launches_per_step = (step, None) if args.eager else ctx.capture(step)
    run()
    torch.cuda.synchronize()
    with ClockSampler(ctx.dev_index) as clk:
        ms = ctx.timed(run, args.steps)
    total_ms = ctx.max_over_ranks(sum(ms))
    value = K * NT * args.steps / (total_ms / 1e3)          # stage-DAG scorings, all ranks
    searches = len(Bs) * args.steps / (total_ms / 1e3)
    plans = sts.search.plans()
    # e2e: the stage DAGs' inputs from pinned host memory every step, T* and plans back
    db = sts.db
    pin = None
    if db is not None:
        loc = sts.local
        pin = {"node_ptr": torch.from_numpy(loc.node_ptr).pin_memory(),
               "edge_ptr": torch.from_numpy(loc.edge_ptr).pin_memory(),
               "src": torch.from_numpy(loc.src).pin_memory(), "dst": torch.from_numpy(loc.dst).pin_memory(),
               "feats": torch.from_numpy(np.ascontiguousarray(loc.feats).view(np.uint8).reshape(-1).copy()).pin_memory()}
    outs = [torch.empty(len(Bs), dtype=torch.float64).pin_memory(),
            torch.empty((len(Bs), nl), dtype=torch.int32).pin_memory(),
            torch.empty((len(Bs), nl), dtype=torch.int32).pin_memory(),
            torch.empty(len(Bs), dtype=torch.int32).pin_memory()]

    def e2e_step():
        if pin is not None:
            for k_, t_ in pin.items():
                getattr(db, k_ if k_ != "feats" else "feats").copy_(t_, non_blocking=True)
        step()
        outs[0].copy_(sts.search.T, non_blocking=True)
        outs[1].copy_(sts.search.ends, non_blocking=True)
        outs[2].copy_(sts.search.choices, non_blocking=True)
        outs[3].copy_(sts.search.S, non_blocking=True)

    e2e_run = e2e_step if args.eager else ctx.capture(e2e_step)[0]
    e2e_run()
    ms_e2e = ctx.timed(e2e_run, max(5, args.steps // 2))
    tot_e2e = ctx.max_over_ranks(sum(ms_e2e))
    e2e_value = K * NT * len(ms_e2e) / (tot_e2e / 1e3)
    h2d = ctx.sum_over_ranks(sum(t.numel() * t.element_size() for t in pin.values()) if pin else 0) / max(world, 1)
    d2h = sum(t.numel() * t.element_size() for t in outs)
    prof = ctx.profile(step, max(3, args.steps // 4))
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        import oracle
        oracle.build()
        cores = host_cores()
        gs = list(range(0, NT, max(1, NT // (2 * cores))))[:2 * cores]
        t0 = time.perf_counter()
        oracle.forward_batch(cfgs[0], blobs[0], host, graphs=gs, threads=cores)
        wall = time.perf_counter() - t0
        # one oracle forward per (stage, choice); rate in stage-DAG scorings/s
        cpu = {"value": len(gs) / wall, "unit": UNIT, "cores": cores, "kind": "oracle",
               "sample": f"{len(gs)} of the {NT} layer-range stages (every {max(1, NT // (2 * cores))}th, "
                         f"{min(host.sizes[gs])}-{max(host.sizes[gs])} nodes) on one mesh model, fp64 C "
                         f"oracle, {cores} threads, {wall:.1f} s; the plan search itself is not timed"}
    if rank == 0:
        for k in prof:
            prof[k]["share"] = prof[k]["ms_per_step"] / (total_ms / args.steps)
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "f16", "data": "synthetic",
                "config": {"workload": f"search: all {NT} layer-range stages of GPT-3 1.3B ({nl} layers, Table IV; "
                                       f"{int(host.sizes.min())}-{int(host.sizes.max())} nodes) x {K} mesh models "
                                       f"(Table III), stage table all-reduce, plan search on 4 GPUs (Platform 2) "
                                       f"for B in {Bs}",
                           "stages": NT, "mesh_choices": K, "choice_devices": devs, "cluster_devices": 4,
                           "microbatches": Bs,
                           "parallelism": f"stage-sharded x{world} (cost-balanced), sum-all-reduce of the stage table",
                           "l2": "not flushed: one step's inputs and activations (~0.4 GB) exceed the 126 MB L2",
                           "dagra_k": args.hops if args.hops > 0 else "inf",
                           "layers": cfgs[0]["num_layers"], "d_model": cfgs[0]["d_model"],
                           "heads": cfgs[0]["num_heads"], "d_ff": cfgs[0]["d_ff"]},
                "searches_per_s": searches,
                "best_plans": {str(B): {"T": T, "stages": st} for B, (T, st) in zip(Bs, plans)},
                "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
                        "d2h_bytes_per_step": int(d2h)},
                "gpu_launches": int((launches_per_step or 0) * args.steps),
                "launch_mode": "eager" if args.eager or getattr(ctx, "capture_failed", False) else "cuda_graph",
                "roofline": None, "cpu_baseline": cpu, "clocks": clk.summary(),
                "kernels": {k: {kk: round(vv, 5) for kk, vv in v.items()} for k, v in prof.items()}}
        emit(line, args)


def run_sweep(args, ctx, pool):
    """configs[4]: an owned-mode plan sweep of args.plans plans, cost-balanced
    over the ranks (strong scaling: the total is fixed).  One step = build +
    forward of every stage graph of the rank's plans (chunks of args.chunk),
    Eqn 4 over its plans, all-gather of T, global argmin."""
    import torch
    from paper_conf_ipps_acharyas25_b200 import synth, sweep
    pt, L, dev, world, rank = ctx.pt, ctx.L, ctx.dev, ctx.world, ctx.rank

    cfg = dict(synth.MODEL_CONFIGS["gpt"], _name="gpt")
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    (p0, p1), pp, mb, s0, counts = sweep.shard_sweep(args.plans, world, rank)
    model = pt.Model(cfg, blob, device=dev)
    sh = sweep.SweepShard(pt, model, pool, pp, mb, s0, chunk=args.chunk, device=dev)
    Pmax = max(counts)
    T_pad = torch.full((Pmax,), float("inf"), dtype=torch.float64, device=dev)
    T_all = torch.empty(world * Pmax, dtype=torch.float64, device=dev)
    best = torch.empty(1, dtype=torch.int64, device=dev)
    # global plan id of padded slot r*Pmax + i is (start of rank r) + i; padding is +inf, never chosen
    # unless every T is inf; the argmin below maps the padded index back.
    starts = np.concatenate([[0], np.cumsum(counts)])[:-1]

    def step():
        T = sh.score()
        if world > 1:
            T_pad[:sh.num_plans].copy_(T)
            ctx.all_gather_T(T_all, T_pad)
            pt.predtop_plan_argmin(T_all, best)
        else:
            pt.predtop_plan_argmin(T, best)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    st, bad = sh.status()
    assert st == pt.OK, (st, bad)
    assert torch.isfinite(sh.lat).all()

    # CUDA-graph capture of the whole sweep step (~125 chunk builds + forwards):
    # eager, the step is bound by host enqueue, not by the kernels
    capture = not (args.eager or ctx.gloo)
    launches_per_step = None
    run = step
    if capture:
        run, launches_per_step = ctx.capture(step)
        run()
        torch.cuda.synchronize()
    launches0 = L.predtop_launch_count()
    with ClockSampler(ctx.dev_index) as clk:
        ms = ctx.timed(run, args.steps, flush=False)
    launches = L.predtop_launch_count() - launches0
    if launches_per_step is not None:
        launches = launches_per_step * args.steps
    total_ms = ctx.max_over_ranks(sum(ms))
    graphs_total = ctx.sum_over_ranks(float(sh.num_stages))
    value = graphs_total * args.steps / (total_ms / 1e3)
    plans_per_s = args.plans * args.steps / (total_ms / 1e3)
    b = int(best.item())
    if world > 1:  # padded index -> global plan id
        r, i = divmod(b, Pmax)
        b = int(starts[r] + i)
    else:
        b += p0

    # ---- e2e: every chunk's inputs copied from pinned host memory before its build
    pins = {}
    for key, db in sh.batches.items():
        pins[key] = [(getattr(db, n), getattr(db, n).cpu().pin_memory())
                     for n in ("node_ptr", "edge_ptr", "src", "dst", "feats")]
    plan_pin = [(sh.plans.plan_ptr, sh.plans.plan_ptr.cpu().pin_memory()),
                (sh.plans.plan_stage, sh.plans.plan_stage.cpu().pin_memory()),
                (sh.plans.microbatches, sh.plans.microbatches.cpu().pin_memory())]
    T_host = torch.empty(max(world * Pmax, 1), dtype=torch.float64).pin_memory()
    h2d = sum(h.numel() * h.element_size() for _, _, k in sh.chunks for _, h in pins[k]) + \
        sum(h.numel() * h.element_size() for _, h in plan_pin)
    d2h = (world * Pmax if world > 1 else sh.num_plans) * 8 + 8

    # the H2D copy of chunk c+1 runs on a copy stream while chunk c is scored;
    # chunks share device buffer sets (SweepShard keys them by pool offset and
    # size), so a copy into set `key` first waits for the forward of the last
    # chunk that read that set (write-after-read); when chunk c+1 reuses chunk
    # c's own set, its copy is issued only after chunk c's forward
    cs = torch.cuda.Stream(device=dev)
    evs = [torch.cuda.Event() for _ in sh.chunks]
    done = [torch.cuda.Event() for _ in sh.chunks]

    def e2e_step():
        cur = torch.cuda.current_stream()
        cs.wait_stream(cur)
        last_user = {}

        def copy_chunk(c):
            key = sh.chunks[c][2]
            with torch.cuda.stream(cs):
                if key in last_user:
                    cs.wait_event(done[last_user[key]])
                for dev_t, host_t in pins[key]:
                    dev_t.copy_(host_t, non_blocking=True)
                evs[c].record(cs)

        with torch.cuda.stream(cs):
            for dev_t, host_t in plan_pin:
                dev_t.copy_(host_t, non_blocking=True)
        copy_chunk(0)
        n = len(sh.chunks)
        for c, (lo, hi, key) in enumerate(sh.chunks):
            early = c + 1 < n and sh.chunks[c + 1][2] != key
            if early:
                copy_chunk(c + 1)
            cur.wait_event(evs[c])
            sh.dags[key].rebuild()
            sh.model.forward(sh.dags[key], sh.ws, sh.lat[lo:hi])
            done[c].record(cur)
            last_user[key] = c
            if c + 1 < n and not early:
                copy_chunk(c + 1)
        cur.wait_stream(cs)
        T, _, _ = sh.plans.latency(sh.lat, no_sync=True)
        if world > 1:
            T_pad[:sh.num_plans].copy_(T)
            ctx.all_gather_T(T_all, T_pad)
            pt.predtop_plan_argmin(T_all, best)
            T_host.copy_(T_all, non_blocking=True)
        else:
            pt.predtop_plan_argmin(T, best)
            T_host[:sh.num_plans].copy_(T, non_blocking=True)

    e2e_run = ctx.capture(e2e_step)[0] if capture else e2e_step
    e2e_run()
    ms_e2e = ctx.timed(e2e_run, max(2, args.steps // 2), flush=False)
    tot_e2e = ctx.max_over_ranks(sum(ms_e2e))
    e2e_value = graphs_total * len(ms_e2e) / (tot_e2e / 1e3)

    prof = ctx.profile(step, 2)
    nodes = sum(sh.batches[k].total_nodes for _, _, k in sh.chunks)
    edges = sum(sh.batches[k].total_edges for _, _, k in sh.chunks)
    words, A = 0, 0
    for key, dag in sh.dags.items():
        sizes = np.diff(sh.batches[key].node_ptr.cpu().numpy())
        uses = sum(1 for _, _, k in sh.chunks if k == key)
        words += uses * int(sum(n * 2 * ((n + 127) // 128) for n in sizes))
        A += uses * dag_pairs(pt, dag, sizes)
    work = algorithmic_work(cfg, nodes, edges, words, A)
    roof = roofline(prof, work, cfg, A, nodes, clk, total_ms / args.steps)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        host = synth.pack_graphs(list(pool[:1024]))
        v, cores, n, wall, _ = oracle_rate(cfg, blob, host)
        cpu = {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle",
               "sample": f"first {n} pool stage graphs, fp64 C oracle, {cores} threads, {wall:.1f} s"}
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "f16", "data": "synthetic",
                "config": workload_config(args),
                "plans_per_s": plans_per_s, "graphs_per_step": graphs_total, "best_plan": b,
                "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
                        "d2h_bytes_per_step": int(d2h)},
                "gpu_launches": int(launches),
                "launch_mode": "eager" if not capture or getattr(ctx, "capture_failed", False) else "cuda_graph",
                "roofline": roof, "cpu_baseline": cpu, "clocks": clk.summary(),
                "kernels": {k: {kk: round(vv, 5) for kk, vv in v.items()} for k, v in prof.items()}}
        emit(line, args)


def run_train(args, ctx):
    """training steps of the paper's model (4 DAG-
    Transformer layers of width 64, mini-batches of 32 stage graphs, MAE loss,
    Adam) on GPT-style stage DAGs.  One step = predtop_train_grad (fp32
    forward, loss, backward) + predtop_train_adam on one mini-batch per rank;
    with N ranks the gradients are averaged by one NCCL all-reduce before
    Adam (data-parallel training: the one real exchange of this path)."""
    import torch
    from paper_conf_ipps_acharyas25_b200 import synth
    pt, dev, world, rank = ctx.pt, ctx.dev, ctx.world, ctx.rank
    cfg = dict(synth.MODEL_CONFIGS["paper"])
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    G = args.graphs
    host = synth.stage_batch("gpt", G, first_graph=rank * G)
    # labels: any latency-like targets (throughput does not depend on them)
    y_host = (0.01 * np.diff(host.node_ptr).astype(np.float32) + 1.0)
    y_pin = torch.from_numpy(y_host).pin_memory()
    y = torch.empty(G, dtype=torch.float32, device=dev)
    y.copy_(y_pin)
    tr = pt.Trainer(cfg, blob, device=dev)
    dag = pt.Dag(pt.DeviceBatch.from_host(host, device=dev))
    grad = tr.buffer(pt.Trainer.GRAD)

    def step():
        tr.grad(dag, y)
        if world > 1:
            if ctx.gloo:
                g = grad.cpu()
                ctx.dist.all_reduce(g)
                grad.copy_(g)
            else:
                ctx.dist.all_reduce(grad)
            grad.mul_(1.0 / world)
        tr.adam(1e-3)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    l0 = ctx.L.predtop_launch_count()
    step()
    torch.cuda.synchronize()
    launches = ctx.L.predtop_launch_count() - l0
    with ClockSampler(ctx.dev_index) as clk:
        ms = ctx.timed(step, args.steps)
    total_ms = ctx.max_over_ranks(sum(ms))
    value = world * G * args.steps / (total_ms / 1e3)
    loss_pin = torch.empty(1, dtype=torch.float32).pin_memory()

    def e2e_step():  # labels in from pinned host memory, loss back, every step
        y.copy_(y_pin, non_blocking=True)
        loss, _ = tr.grad(dag, y)
        if world > 1:
            if ctx.gloo:
                g = grad.cpu()
                ctx.dist.all_reduce(g)
                grad.copy_(g)
            else:
                ctx.dist.all_reduce(grad)
            grad.mul_(1.0 / world)
        tr.adam(1e-3)
        loss_pin.copy_(loss, non_blocking=True)

    e2e_ms = ctx.max_over_ranks(sum(ctx.timed(e2e_step, args.steps)))
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        import time
        import oracle
        oracle.build()
        cores = host_cores()
        n = min(G, max(cores, 16))
        sub = host.subset(list(range(n)))
        t0 = time.perf_counter()
        oracle.mae_grad(cfg, blob, sub, y_host[:n], threads=cores)
        wall = time.perf_counter() - t0
        cpu = {"value": n / wall, "unit": "graphs/s", "cores": cores, "kind": "oracle",
               "sample": f"{n} of the {G} stage graphs: fp64 forward + MAE gradient (orc_grad), {cores} threads, {wall:.1f} s"}
    if rank == 0:
        line = {"metric": "stage-DAGs trained/sec (forward + MAE + backward + Adam)", "value": value,
                "unit": "graphs/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": total_ms / args.steps, "higher_is_better": True, "scaling": "weak",
                "vs_baseline": None, "dtype": "f32", "data": "synthetic",
                "config": {"workload": f"train: mini-batches of {G} GPT-style stage DAGs (~300 ops) per GPU, paper "
                                       "model (4 layers, d=64, 4 heads, d_ff=256; P:178), MAE loss, Adam; "
                                       "data-parallel gradient all-reduce for N > 1",
                           "graphs_per_gpu": G, "l2": "flushed before every timed step (256 MiB memset, untimed)"},
                "e2e": {"value": world * G * args.steps / (e2e_ms / 1e3), "unit": "graphs/s",
                        "h2d_bytes_per_step": 4 * G, "d2h_bytes_per_step": 4},
                "gpu_launches": int(launches), "cpu_baseline": cpu, "launch_mode": "eager",
                "clocks": clk.summary()}
        emit(line, args)


def emit(line, args):
    print(json.dumps(line), flush=True)
    if args.profile_json:
        with open(args.profile_json, "w") as f:
            json.dump(line, f, indent=1)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="moe", choices=["tiny", "gpt", "moe", "16k", "sweep", "search", "train"])
    ap.add_argument("--no-also", action="store_true",
                    help="moe: skip the configs[1] (GPT) measurement reported under 'also'")
    ap.add_argument("--no-extras", action="store_true",
                    help="time the step only (no e2e, profile, cpu_baseline); the line carries the T hash")
    ap.add_argument("--layers", type=int, default=24, help="search: model layers (GPT-3 1.3B: 24)")
    ap.add_argument("--graphs", type=int, default=None, help="stage graphs per GPU (default per config)")
    ap.add_argument("--plans", type=int, default=100000, help="sweep: total candidate plans")
    ap.add_argument("--chunk", type=int, default=4096, help="sweep: stage graphs per build+forward launch")
    ap.add_argument("--pool", type=int, default=8192, help="sweep: distinct synthetic stage graphs")
    ap.add_argument("--hops", type=int, default=0,
                    help="DAGRA range k (P:145): 0 = infinity (the paper's setting); k >= 1 = k-hop mask")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--profile-json", default=None)
    ap.add_argument("--eager", action="store_true", help="no CUDA-graph capture of the step")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo: host-side all-gather (eager only); lets N ranks share one GPU to test the "
                         "multi-rank flow on a 1-GPU box")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.graphs is None:
        args.graphs = DEFAULT_GRAPHS[args.config]

    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        # one process per GPU: re-launch under torch.distributed.run
        import socket
        import subprocess
        with socket.socket() as so:
            so.bind(("127.0.0.1", 0))
            port = so.getsockname()[1]
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
        sys.exit(subprocess.call(cmd))
    rank = int(os.environ.get("RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank)
        return
    pool = None
    if args.config == "sweep":  # host generation before any CUDA context (forked pool)
        from paper_conf_ipps_acharyas25_b200 import synth
        pool = synth.stage_graphs_parallel("gpt", args.pool)
    ctx = Ctx(args)
    if args.config == "sweep":
        run_sweep(args, ctx, pool)
    elif args.config == "search":
        run_search(args, ctx)
    elif args.config == "train":
        run_train(args, ctx)
    else:
        line = run_batch(args, ctx)
        if args.config == "moe" and not args.no_also and not args.no_extras:
            import copy
            a2 = copy.copy(args)
            a2.config, a2.graphs, a2.steps = "gpt", DEFAULT_GRAPHS["gpt"], max(10, args.steps // 2)
            a2.profile_json = None
            l2 = run_batch(a2, ctx)
            if line is not None and l2 is not None:
                line["also"] = {"gpt": {k: l2[k] for k in ALSO_KEYS if k in l2}}
        if line is not None:
            emit(line, args)
    ctx.finish()


if __name__ == "__main__":
    main()
