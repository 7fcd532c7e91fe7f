"""Latency of a fixed GPT batch in this process: prints a digest and the max
relative error vs the oracle (used to check cross-process repeatability)."""
import hashlib, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
from paper_conf_ipps_acharyas25_b200 import predtop as pt, synth
cfg = synth.MODEL_CONFIGS["gpt"]
blob = synth.pack_weights(cfg, synth.model_weights(cfg))
b = synth.stage_batch("gpt", 24)
m = pt.Model(cfg, blob)
dag = pt.Dag(pt.DeviceBatch.from_host(b))
y = m.forward(dag).cpu().numpy().astype(np.float64)
want = oracle.forward_batch(cfg, blob, b)
err = np.abs(y - want) / np.abs(want)
print(hashlib.md5(y.tobytes()).hexdigest()[:12], "max rel err %.3e argmax %d" % (err.max(), err.argmax()))
