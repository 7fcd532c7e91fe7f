"""Timeline of the layer-tail v2 kernel (k_layer_tail2, CTA 0, first tiles)
from the PREDTOP_TRACE debug build.
Usage: PREDTOP_LIB=.../libpredtop_trace.so python tools/tail2_trace.py"""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_acharyas25_b200 import predtop as pt, synth  # noqa: E402

NAMES = ["start", "x loaded", "o_full", "LN1 done", "f0", "f1", "f2", "f3", "p0", "p1", "p2", "p3",
         "out_full", "LN2 done", "stored"]


def main():
    cfg = synth.MODEL_CONFIGS["gpt"]
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    host = synth.stage_batch("gpt", 1024)
    m = pt.Model(cfg, blob)
    dag = pt.Dag(pt.DeviceBatch.from_host(host), no_sync=True)
    ws = m.forward_workspace(dag)
    lat = torch.empty(1024, device="cuda")
    for _ in range(3):
        m.forward(dag, ws, lat)
    torch.cuda.synchronize()
    buf = (ctypes.c_ulonglong * 264)()
    pt.lib().predtop_debug_tail2_trace.argtypes = [ctypes.c_void_p]
    assert pt.lib().predtop_debug_tail2_trace(ctypes.cast(buf, ctypes.c_void_p)) == 0
    raw = np.frombuffer(buf, dtype=np.uint64).astype(np.int64)
    t = raw[:256].reshape(16, 16)
    mw = raw[256:264]
    t0 = t[0, 0]
    ntile = int((t[:, 0] > 0).sum())
    print("tile " + " ".join(f"{n:>9s}" for n in NAMES))
    for i in range(ntile):
        print(f"{i:4d} " + " ".join(f"{(t[i, k] - t0) / 1000:9.2f}" for k in range(15)))
    d = np.diff(t[1:ntile, :15], axis=1).mean(0) / 1000
    print("mean phase durations (us):", " ".join(f"{NAMES[k + 1]}:{d[k]:.2f}" for k in range(14)))
    print("tile period (us): %.2f" % (np.diff(t[1:ntile, 0]).mean() / 1000))
    print("MMA thread, mean per tile over tiles 2..9 (clk): ring_full wait %d, o_empty wait %d, h_ready wait %d, "
          "p_ready wait %d, tile span %d" % tuple(mw[:5] // 8))


if __name__ == "__main__":
    main()
