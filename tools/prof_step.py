"""Run W warm-up steps + K steps of the bench workload (no timing, no extras):
the target for ncu launch lists and --set full captures.
Usage: python tools/prof_step.py [--config gpt] [--graphs 1024] [--warmup 2] [--steps 1]"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="gpt")
    ap.add_argument("--graphs", type=int, default=1024)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--steps", type=int, default=1)
    a = ap.parse_args()
    import torch
    from paper_conf_ipps_acharyas25_b200 import build, predtop as pt, synth
    build.build_library()
    cfg = synth.MODEL_CONFIGS[a.config]
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    host = synth.stage_batch(a.config, a.graphs)
    ps = synth.owned_plans(a.graphs, 4, 16)
    model = pt.Model(cfg, blob)
    dag = pt.Dag(pt.DeviceBatch.from_host(host), no_sync=True)
    ws = model.forward_workspace(dag)
    lat = torch.empty(a.graphs, dtype=torch.float32, device="cuda")
    plans = pt.Plans(ps.plan_ptr, ps.plan_stage, ps.microbatches)
    for _ in range(a.warmup + a.steps):
        dag.rebuild()
        model.forward(dag, ws, lat)
        T, _, _ = plans.latency(lat, no_sync=True)
        plans.argmin(T)
    torch.cuda.synchronize()
    print("launches per step:", pt.launch_count() // (a.warmup + a.steps))


if __name__ == "__main__":
    main()
