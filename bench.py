#!/usr/bin/env python
"""bench.py -- PredTOP prediction path on B200 (BASELINE.json configs[1]).

One step = the whole hot path over one batch: predtop_build_dag (validate,
depth, closure, mask) + predtop_stage_forward (DAG-Transformer, 4 layers) +
predtop_plan_latency (Eqn 4) + [N>1: NCCL all-gather of plan latencies] +
predtop_plan_argmin.  Workload per GPU: 1024 GPT-style stage DAGs of 270-330
ops (seeded, synthetic), d=128, 8 heads, d_ff=512; 256 plans of 4 stages x 16
microbatches (owned mode).  Weak scaling: rank r scores graphs
[1024 r, 1024 (r+1)).

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


def oracle_rate(cfg, blob, batch, target_s: float = 15.0, max_graphs: int = 1024):
    """Oracle graphs/s on a bounded sample with all host cores."""
    import oracle
    oracle.build()
    cores = host_cores()
    t0 = time.perf_counter()
    oracle.forward_batch(cfg, blob, batch, graphs=[0], threads=1)
    t1 = time.perf_counter() - t0
    n = int(max(cores, min(max_graphs, batch.num_graphs, round(target_s * cores / max(t1, 1e-6)))))
    n = min(n, batch.num_graphs)
    t0 = time.perf_counter()
    oracle.forward_batch(cfg, blob, batch, graphs=list(range(n)), threads=cores)
    wall = time.perf_counter() - t0
    return n / wall, cores, n, wall


def run_reference(args, rank):
    if rank != 0:
        return
    from paper_conf_ipps_acharyas25_b200 import synth
    import oracle
    oracle.build()
    cfg = synth.MODEL_CONFIGS[args.config]
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    cores = host_cores()
    per_step = cores  # one graph per core per step
    batch = synth.stage_batch(args.config, per_step * (args.warmup + args.steps) if args.steps * per_step <= 4096 else 4096)
    plans_B = 16
    done, t_total = 0, 0.0
    for s in range(args.warmup + args.steps):
        gs = [(s * per_step + i) % batch.num_graphs for i in range(per_step)]
        t0 = time.perf_counter()
        y = oracle.forward_batch(cfg, blob, batch, graphs=gs, threads=cores)
        # plan formula over the sampled stages (owned mode, 4 stages x B = 16)
        P = len(gs) // 4
        if P:
            oracle.plan_T(np.arange(P + 1) * 4, np.arange(4 * P), np.full(P, plans_B), y[:4 * P].astype(np.float32))
        dt = time.perf_counter() - t0
        if s >= args.warmup:
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


def workload_config(args):
    return {"workload": f"{args.config}: {args.graphs} stage DAGs/GPU x 270-330 ops (fwd+bwd GPT-3 stage "
                        f"template), DAG-Transformer 4 layers d=128 H=8 d_ff=512, sum pool + MLP head; "
                        f"{args.graphs // 4} plans x 4 stages x B=16 (Eqn 4)",
            "graphs_per_gpu": args.graphs, "plans_per_gpu": args.graphs // 4, "stages_per_plan": 4,
            "microbatches": 16, "layers": 4, "d_model": 128, "heads": 8, "d_ff": 512,
            "parallelism": f"graph-sharded x{args.gpus} (owned plans), NCCL all-gather of plan latencies",
            "l2": "flushed before every timed step (256 MiB memset, untimed)",
            "precision": "f16 MMA operands, f32 accumulate/softmax/LN/residual, f32 latency, f64 Eqn 4"}


# ----------------------------------------------------------------- main leg
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="gpt")
    ap.add_argument("--graphs", type=int, default=1024)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--profile-json", default=None)
    ap.add_argument("--eager", action="store_true", help="no CUDA-graph capture of the step")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo: host-side all-gather (eager only); lets N ranks share one GPU to test the "
                         "multi-rank flow on a 1-GPU box")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank)
        return

    import torch
    import torch.distributed as dist
    from paper_conf_ipps_acharyas25_b200 import build, predtop as pt, synth

    gloo = args.dist_backend == "gloo"
    if gloo:
        args.eager = True  # a host-side collective cannot sit inside a CUDA graph
    dev_index = local % torch.cuda.device_count() if gloo else local
    torch.cuda.set_device(dev_index)
    dev = torch.device("cuda", dev_index)
    if world > 1:
        if gloo:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
    if rank == 0:
        build.build_library()
    if world > 1:
        dist.barrier()
    L = pt.lib()
    stream = torch.cuda.current_stream()

    cfg = synth.MODEL_CONFIGS[args.config]
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    G = args.graphs
    host = synth.stage_batch(args.config, G, first_graph=rank * G)
    ps = synth.owned_plans(G, 4, 16)
    model = pt.Model(cfg, blob, device=dev)
    db = pt.DeviceBatch.from_host(host, device=dev)
    dag = pt.Dag(db, no_sync=True)
    ws = model.forward_workspace(dag)
    lat = torch.empty(G, dtype=torch.float32, device=dev)
    plans = pt.Plans(ps.plan_ptr, ps.plan_stage, ps.microbatches, device=dev)
    P = plans.num_plans
    T_all = torch.empty(world * P, dtype=torch.float64, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    def step():
        dag.rebuild()                       # predtop_build_dag (NO_SYNC)
        model.forward(dag, ws, lat)         # predtop_stage_forward
        T, _, _ = plans.latency(lat, no_sync=True)   # predtop_plan_latency
        if world > 1:
            if gloo:
                parts = [torch.empty(P, dtype=torch.float64) for _ in range(world)]
                dist.all_gather(parts, T.cpu())
                T_all.copy_(torch.cat(parts))
            else:
                dist.all_gather_into_tensor(T_all, T)
            plans.argmin(T_all)             # global argmin by (T, global plan id)
        else:
            plans.argmin(T)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    st, bad = dag.dag_status()
    assert st == pt.OK, (st, bad)
    assert torch.isfinite(lat).all()

    def timed(fn, k):
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(k)]
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        for a, b in evs:
            flush.zero_()
            a.record(stream)
            fn()
            b.record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        return [a.elapsed_time(b) for a, b in evs]

    def max_over_ranks(x):
        if world > 1:
            t = torch.tensor([x], dtype=torch.float64, device="cpu" if gloo else dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            return float(t.item())
        return x

    # eager diagnostics: host enqueue time of one step and eager device time
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(5):
        step()
    host_enqueue_ms = (time.perf_counter() - t0) / 5 * 1e3
    torch.cuda.synchronize()
    eager_ms = sum(timed(step, 5)) / 5

    # The step is captured once as a CUDA graph (library calls are capturable:
    # NO_SYNC build, stream-ordered kernels, NCCL all-gather) and replayed.
    graph = None
    launches_per_step = None
    if not args.eager:
        side = torch.cuda.Stream(device=dev)
        side.wait_stream(stream)
        with torch.cuda.stream(side):
            step()
        stream.wait_stream(side)
        torch.cuda.synchronize()
        graph = torch.cuda.CUDAGraph()
        l0 = L.predtop_launch_count()
        with torch.cuda.graph(graph, stream=side):
            step()
        launches_per_step = L.predtop_launch_count() - l0
        torch.cuda.synchronize()
        run = graph.replay
    else:
        run = step
    run()
    torch.cuda.synchronize()

    launches0 = L.predtop_launch_count()
    with ClockSampler(dev_index) as clk:
        ms = timed(run, args.steps)
    launches = L.predtop_launch_count() - launches0
    if graph is not None:
        launches = launches_per_step * args.steps
    total_ms = max_over_ranks(sum(ms))
    value = world * G * args.steps / (total_ms / 1e3)
    plans_per_s = world * P * args.steps / (total_ms / 1e3)
    # the replayed step computed the same results as the eager one
    assert torch.isfinite(lat).all()

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
    T_host = torch.empty(world * P, dtype=torch.float64).pin_memory()
    best_host = torch.empty(1, dtype=torch.int64).pin_memory()
    h2d = sum(t.numel() * t.element_size() for t in pin.values())
    d2h = T_host.numel() * 8 + 8

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
        T_host.copy_(T_all if world > 1 else plans.T[:P], non_blocking=True)
        best_host.copy_(plans.best, non_blocking=True)

    e2e_run = e2e_step
    if not args.eager:
        side = torch.cuda.Stream(device=dev)
        side.wait_stream(stream)
        with torch.cuda.stream(side):
            e2e_step()
        stream.wait_stream(side)
        torch.cuda.synchronize()
        g2 = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g2, stream=side):
            e2e_step()
        e2e_run = g2.replay
    for _ in range(2):
        e2e_run()
    ms_e2e = timed(e2e_run, max(10, args.steps // 4))
    tot_e2e = max_over_ranks(sum(ms_e2e))
    e2e_value = world * G * len(ms_e2e) / (tot_e2e / 1e3)
    # the host copy of the plan latencies matches the device result
    torch.cuda.synchronize()
    assert torch.equal(T_host, (T_all if world > 1 else plans.T[:P]).cpu())

    # ---- per-kernel profile pass (separate from the headline timing)
    L.predtop_profile_enable(1)
    prof_steps = max(5, args.steps // 4)
    ms_prof = timed(step, prof_steps)
    L.predtop_profile_enable(0)
    import ctypes
    kinds = 32
    kms = (ctypes.c_double * kinds)()
    kcnt = (ctypes.c_int64 * kinds)()
    nk = L.predtop_profile_read(kms, kcnt, kinds)
    names = [L.predtop_profile_kind_name(i).decode() for i in range(nk)]
    prof = {names[i]: {"ms_per_step": kms[i] / prof_steps, "launches_per_step": kcnt[i] / prof_steps}
            for i in range(nk) if kcnt[i]}
    step_ms_prof = total_ms / args.steps  # shares relative to the headline (graph) step time
    for k in prof:
        prof[k]["share"] = prof[k]["ms_per_step"] / step_ms_prof

    # algorithmic work per launch of each kind
    d, dff, H = cfg["d_model"], cfg["d_ff"], cfg["num_heads"]
    Ntot = host.node_ptr[-1]
    sizes = host.sizes
    T_ = (sizes + 127) // 128
    _, pairs = dag.tiles(int((T_ * T_).sum()))
    A = int(pairs.sum().item())
    E = int(host.edge_ptr[-1])
    words = int(sum(n * 2 * ((n + 127) // 128) for n in sizes))
    work = {
        "gemm_qkv": ("tensor", 2.0 * Ntot * d * 3 * d),
        "gemm_oproj_ln": ("tensor", 2.0 * Ntot * d * d),
        "gemm_ffn1": ("tensor", 2.0 * Ntot * d * dff),
        "gemm_ffn2_ln": ("tensor", 2.0 * Ntot * dff * d),
        "layer_tail": ("tensor", 2.0 * Ntot * (d * d + 2 * d * dff)),
        "attention": ("alu", float(H) * A),  # exps per launch (MUFU-bound)
        "dag_closure": ("hbm", 8.0 * words + 8.0 * E),
        "dag_mask": ("hbm", 3 * 8.0 * words),
        "readout": ("hbm", 4.0 * Ntot * d),
        "embed": ("hbm", Ntot * (20.0 + 4 + 6 * d)),
    }
    peaks, peak_src = load_peaks()
    dom = max(prof, key=lambda k: prof[k]["ms_per_step"]) if prof else None
    roof = None
    if dom in work:
        bound, units = work[dom]
        per_launch_ms = prof[dom]["ms_per_step"] / prof[dom]["launches_per_step"]
        sec = per_launch_ms / 1e3
        if bound == "tensor":
            ach = units / sec / 1e12
            peak = peaks["bf16_tflops_sustained"] if "bf16_tflops_sustained" in peaks else peaks["bf16_tflops"]
            roof = {"bound": "tensor", "achieved": ach, "peak": peak, "unit": "TFLOP/s", "frac": ach / peak}
        elif bound == "hbm":
            ach = units / sec / 1e9
            roof = {"bound": "hbm", "achieved": ach, "peak": peaks["hbm_gbs"], "unit": "GB/s",
                    "frac": ach / peaks["hbm_gbs"]}
        else:
            clk_mhz = (clk.summary()["sm_mhz"] or peaks.get("sm_max_mhz", 1965.0))
            peak = MUFU_EX2_PER_CLK_SM * NUM_SMS * clk_mhz * 1e6 / 1e9
            ach = units / sec / 1e9
            tflops = 4.0 * d * A / sec / 1e12
            roof = {"bound": "alu", "achieved": ach, "peak": peak, "unit": "Gexp/s", "frac": ach / peak,
                    "peak_basis": f"MUFU ex2 {MUFU_EX2_PER_CLK_SM}/clk/SM x {NUM_SMS} SMs x {clk_mhz:.0f} MHz (median under load)",
                    "tensor_equiv_tflops": tflops,
                    "tensor_frac": tflops / peaks.get("bf16_tflops_sustained", peaks["bf16_tflops"])}
        traffic = None
        try:  # DRAM bytes per launch of the dominant kernel from a committed ncu capture
            with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
                tr = json.load(f).get(dom)
            if tr:
                traffic = tr["bytes"]
                roof["traffic_source"] = tr["source"]
                if dom == "attention":  # algorithmic bytes: q,k,v in (3d fp16) + att out (d fp16) per node
                    roof["traffic_algorithmic"] = float(Ntot) * 4 * d * 2
        except (OSError, ValueError, KeyError):
            traffic = None
        roof.update({"kernel": dom, "traffic": traffic, "peak_source": peak_src,
                     "kernel_ms": per_launch_ms, "share_of_step": prof[dom]["share"]})

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        v, cores, n, wall = oracle_rate(cfg, blob, host)
        cpu = {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle",
               "sample": f"first {n} of {G} {args.config} stage graphs, fp64 C oracle, {cores} threads, {wall:.1f} s"}

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "f16", "data": "synthetic",
                "config": workload_config(args),
                "plans_per_s": plans_per_s,
                "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": int(h2d),
                        "d2h_bytes_per_step": int(d2h)},
                "gpu_launches": int(launches),
                "launch_mode": "eager" if args.eager else "cuda_graph",
                "eager_ms_per_step": eager_ms, "host_enqueue_ms_per_step": host_enqueue_ms,
                "roofline": roof, "cpu_baseline": cpu, "clocks": clk.summary(),
                "kernels": {k: {kk: round(vv, 5) for kk, vv in v.items()} for k, v in prof.items()}}
        print(json.dumps(line), flush=True)
        if args.profile_json:
            with open(args.profile_json, "w") as f:
                json.dump(line, f, indent=1)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
