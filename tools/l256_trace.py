"""Timeline of CTA 0 of the fused d=256 layer tail (PREDTOP_TRACE build):
PREDTOP_LIB=.../libpredtop_trace.so python tools/l256_trace.py"""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_acharyas25_b200 import predtop as pt, synth  # noqa: E402


def main():
    cfg = synth.MODEL_CONFIGS["moe"]
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    host = synth.stage_batch("moe", 512)
    m = pt.Model(cfg, blob)
    dag = pt.Dag(pt.DeviceBatch.from_host(host), no_sync=True)
    ws = m.forward_workspace(dag)
    lat = torch.empty(512, device="cuda")
    for _ in range(2):
        m.forward(dag, ws, lat)
    torch.cuda.synchronize()
    buf = (ctypes.c_ulonglong * 256)()
    pt.lib().predtop_debug_l256_trace.argtypes = [ctypes.c_void_p]
    assert pt.lib().predtop_debug_l256_trace(ctypes.cast(buf, ctypes.c_void_p)) == 0
    t = np.frombuffer(buf, dtype=np.uint64).reshape(16, 16).astype(np.int64)
    t0 = t[0, 0]
    names = ["mma:start", "o_empty", "oproj_issued", "h_ready", "ffn_issued", "epi:o_full", "x_ready", "ln1_stats",
             "h_written", "ffn_done", "out_full", "ln2_done", "ln1_bar", "ln1_passB", "ln2_bar"]
    print("tile " + " ".join(f"{n:>12s}" for n in names))
    for i in range(16):
        print(f"{i:4d} " + " ".join(f"{(t[i, k] - t0) if t[i, k] else 0:12d}" for k in range(len(names))))

    w = (ctypes.c_ulonglong * (16 * 16 * 12))()
    pt.lib().predtop_debug_l256_trace_w.argtypes = [ctypes.c_void_p]
    assert pt.lib().predtop_debug_l256_trace_w(ctypes.cast(w, ctypes.c_void_p)) == 0
    w = np.frombuffer(w, dtype=np.uint64).reshape(16, 16, 12).astype(np.int64) - t0
    ev = ["o_full", "x_ready", "stats", "bar1", "passB", "h_wr", "out_full", "ln2_end", "ln2_bar", "ln2_norm", "ln2_w1", "ln2_w2"]
    for i in range(2, 5):
        print(f"tile {i}: per-warp events (min / median / max over the 16 epilogue warps)")
        for k, n in enumerate(ev):
            col = w[i, :, k]
            print(f"   {n:>9s} {col.min():9d} {int(np.median(col)):9d} {col.max():9d}   argmax warp {int(col.argmax())}")


if __name__ == "__main__":
    main()
