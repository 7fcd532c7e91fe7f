"""Timeline of one CTA (blockIdx 3001) of the tcgen05 attention kernel from
the PREDTOP_TRACE debug build (clock64 cycles).  Usage:
  PREDTOP_LIB=.../libpredtop_trace.so python tools/attn_trace.py [config]"""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_acharyas25_b200 import predtop as pt, synth  # noqa: E402


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "moe"
    cfg = synth.MODEL_CONFIGS[name]
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    G = 512 if name == "moe" else 1024
    host = synth.stage_batch(name, G)
    m = pt.Model(cfg, blob)
    dag = pt.Dag(pt.DeviceBatch.from_host(host), no_sync=True)
    ws = m.forward_workspace(dag)
    lat = torch.empty(G, device="cuda")
    for _ in range(3):
        m.forward(dag, ws, lat)
    torch.cuda.synchronize()
    buf = (ctypes.c_ulonglong * (8 * 64))()
    pt.lib().predtop_debug_attn_trace.argtypes = [ctypes.c_void_p]
    assert pt.lib().predtop_debug_attn_trace(ctypes.cast(buf, ctypes.c_void_p)) == 0
    t = np.frombuffer(buf, dtype=np.uint64).reshape(8, 64).astype(np.int64)
    t0 = t[t > 0].min()
    f = lambda x: f"{x - t0:8d}" if x else "       -"
    print("CTA start / barriers+TMEM / m,Qm written / softmax done / O complete / stored:",
          " ".join(f(t[2, i]) for i in range(6)))
    print("chunk | mma: pready_seen  pv_issued  kv_empty_commit | qk: kv_full  issued  s_full_commit | w2: s_seen  arrive")
    for c in range(64):
        if t[0, c] or t[3, c]:
            print(f"{c:4d} | {f(t[0, c])} {f(t[1, c])}        - | {f(t[3, c])} {f(t[4, c])} {f(t[5, c])} | "
                  f"{f(t[6, c])} {f(t[7, c])}")


if __name__ == "__main__":
    main()
