import sys, os; sys.path.insert(0, os.getcwd())
import numpy as np, torch
from paper_conf_ipps_acharyas25_b200 import synth, predtop as pt
host = synth.layer_range_stages("gpt", 24)
db = pt.DeviceBatch.from_host(host); dag = pt.Dag(db)
for c in range(6):
    cfg = dict(synth.MODEL_CONFIGS["search"]); cfg["seed"] += c; cfg["head_scale"] = 1.0; cfg["out_bias"] = 0.0
    m = pt.Model(cfg, synth.pack_weights(cfg, synth.model_weights(cfg)))
    y = m.forward(dag).cpu().numpy()
    n = host.sizes
    print(c, "raw min %.3f max %.3f mean %.3f std %.3f" % (y.min(), y.max(), y.mean(), y.std()),
          "corr(N) %.2f" % np.corrcoef(y, n)[0, 1], "y/N range", (y / n).min(), (y / n).max())
