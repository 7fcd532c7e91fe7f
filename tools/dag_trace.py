"""Phase timing of the fused small-graph DAG build (k_dag_small), graphs 0..63,
from the PREDTOP_TRACE debug build: PREDTOP_LIB=.../libpredtop_trace.so python tools/dag_trace.py"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_acharyas25_b200 import predtop as pt, synth  # noqa: E402


def main():
    host = synth.stage_batch("gpt", 1024)
    dag = pt.Dag(pt.DeviceBatch.from_host(host), no_sync=True)
    torch.cuda.synchronize()
    buf = (ctypes.c_longlong * 9)()
    pt.lib().predtop_debug_dag_trace.argtypes = [ctypes.c_void_p]
    assert pt.lib().predtop_debug_dag_trace(ctypes.cast(buf, ctypes.c_void_p)) == 0
    v = list(buf)
    lv = (v[8] & 0xffffffff) / 64
    names = ["CSR built", "Kahn done", "closure done", "mask done", "end"]
    print(f"mean levels per graph {lv:.1f}; mean clocks from kernel entry (graphs 0..63):")
    for k, n in enumerate(names):
        print(f"  {n:14s} {v[k] / 64:10.0f}")


if __name__ == "__main__":
    main()
