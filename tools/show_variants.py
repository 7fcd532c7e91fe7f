"""Summarise gpurun_out/bench_<v>.json files written by tools/run_variants.sh."""
import glob
import json
import os

for f in sorted(glob.glob("gpurun_out/bench_*.json")):
    v = os.path.basename(f)[6:-5]
    try:
        d = json.load(open(f))
    except Exception as e:  # noqa: BLE001
        print(v, "unreadable", e)
        continue
    k = {n: x["ms_per_step"] for n, x in d.get("kernels", {}).items() if x["ms_per_step"] > 0.04}
    print(f"{v:10s} {d['value']:10.0f} {d['unit']}  {d['ms_per_step']:.3f} ms/step  frac {d['roofline']['frac']:.3f}  {k}")
