"""Timeline of the fused layer-tail kernel (CTA 0) from the PREDTOP_TRACE
debug build.  Usage: PREDTOP_LIB=.../libpredtop_trace.so python tools/tail_trace.py"""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_acharyas25_b200 import predtop as pt, synth  # noqa: E402

NAMES = ["start", "x_free", "o_full", "x_full", "LN1 done", "f0", "r0", "f1", "r1", "f2", "r2", "f3", "r3",
         "out_full", "LN2+store"]


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
    buf = (ctypes.c_ulonglong * 328)()
    pt.lib().predtop_debug_tail_trace.argtypes = [ctypes.c_void_p]
    assert pt.lib().predtop_debug_tail_trace(ctypes.cast(buf, ctypes.c_void_p)) == 0
    raw = np.frombuffer(buf, dtype=np.uint64).astype(np.int64)
    t = raw[:256].reshape(16, 16)
    w = raw[256:320].reshape(4, 16)
    mw = raw[320:328]
    t0 = t[0, 0]
    print("tile " + " ".join(f"{n:>9s}" for n in NAMES))
    for i in range(12):
        print(f"{i:4d} " + " ".join(f"{(t[i, k] - t0) / 1000:9.2f}" for k in range(15)))
    d = np.diff(t[:12, :15], axis=1).mean(0) / 1000
    print("mean phase durations (us):", " ".join(f"{NAMES[k + 1]}:{d[k]:.2f}" for k in range(14)))
    w0 = w[0].min()
    for k, n in enumerate(["after waits", "after tmem_ld", "after stores", "after fences"]):
        print(f"chunk1 tile4 {n:14s} (clk, per epilogue warp):", " ".join(f"{x - w0:6d}" for x in w[k]))
    print("MMA warp, mean per tile (clk): ring_full wait %d, p_ready wait %d, h_ready wait %d, a_full wait %d, "
          "o/out_empty wait %d, tile span %d" % tuple(mw[:6] // 8))


if __name__ == "__main__":
    main()
