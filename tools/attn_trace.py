"""Timeline of one CTA of the tcgen05 attention kernel from the PREDTOP_TRACE
debug build.  Usage: PREDTOP_LIB=.../libpredtop_trace.so python tools/attn_trace.py"""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_acharyas25_b200 import predtop as pt, synth  # noqa: E402


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
    buf = (ctypes.c_ulonglong * 96)()
    pt.lib().predtop_debug_attn_trace.argtypes = [ctypes.c_void_p]
    assert pt.lib().predtop_debug_attn_trace(ctypes.cast(buf, ctypes.c_void_p)) == 0
    t = np.frombuffer(buf, dtype=np.uint64).reshape(6, 16).astype(np.int64)
    t0 = t[0, 0]
    f = lambda x: f"{(x - t0) / 1000:7.2f}" if x else "      -"
    print("mma start/bar_ld/vt_ready:", f(t[0, 0]), f(t[0, 1]), f(t[0, 2]), " vt written", f(t[0, 5]),
          " softmax o_wait begin/end", f(t[0, 3]), f(t[0, 4]), " end", f(t[0, 6]))
    print("chunk  sfull_wait_begin  sfull_seen  p_arrive  mma_pready_seen")
    for c in range(16):
        if t[2, c]:
            print(f"{c:4d}  {f(t[2, c])}  {f(t[3, c])}  {f(t[4, c])}  {f(t[1, c])}")


if __name__ == "__main__":
    main()
