"""Small end-to-end run of every hot-path kernel for compute-sanitizer:
tiny + 2 GPT graphs + 16 MoE-size graphs (187 layer-tail tiles: CTAs run several tiles) through build_dag / stage_forward /
plan_latency, plus one training step (memcheck / racecheck / synccheck)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_acharyas25_b200 import build, predtop as pt, synth  # noqa: E402


def main():
    build.build_library()
    for name, batch in [("tiny", synth.tiny_batch()), ("gpt", synth.stage_batch("gpt", 2)),
                        ("moe", synth.stage_batch("moe", 16))]:
        cfg = synth.MODEL_CONFIGS[name]
        model = pt.Model(cfg, synth.pack_weights(cfg, synth.model_weights(cfg)))
        dag = pt.Dag(pt.DeviceBatch.from_host(batch))
        y = model.forward(dag)
        plans = pt.Plans([0, batch.num_graphs], list(range(batch.num_graphs)), [4])
        T, st, _ = plans.latency(y)
        torch.cuda.synchronize()
        print(name, y.cpu().numpy(), T.cpu().numpy(), flush=True)
    cfg = dict(synth.MODEL_CONFIGS["tiny"])
    tr = pt.Trainer(cfg, synth.pack_weights(cfg, synth.model_weights(cfg)))
    dag = pt.Dag(pt.DeviceBatch.from_host(synth.tiny_batch()))
    loss, _ = tr.grad(dag, torch.ones(4, device="cuda"))
    tr.adam(1e-3)
    torch.cuda.synchronize()
    print("train loss", float(loss.item()))


if __name__ == "__main__":
    main()
