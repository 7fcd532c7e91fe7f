"""Format an ncu --metrics gpu__time_duration.sum --csv launch list (from
tools/prof_step.py --warmup 1 --steps 1) for profiles/: every launch, then
per-kernel totals and shares of the measured step (the last step, from the
last k_meta on).
Usage: python tools/launch_list.py gpurun_out/launches.csv [title]"""
import csv
import re
import sys


def main():
    path = sys.argv[1]
    title = sys.argv[2] if len(sys.argv) > 2 else "GPT config, 1024 graphs"
    hdr, out = None, []
    for r in csv.reader(open(path)):
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d.get("Metric Name") == "gpu__time_duration.sum":
                v = float(d["Metric Value"].replace(",", ""))
                u = d["Metric Unit"]
                us = v / 1000 if u == "ns" else v * 1000 if u == "ms" else v
                out.append((d["Kernel Name"], us))
    metas = [i for i, (k, _) in enumerate(out) if k.startswith("k_meta")]
    step = out[metas[-1]:] if metas else out
    print("# ncu --metrics gpu__time_duration.sum --clock-control none: tools/prof_step.py --warmup 1 --steps 1")
    print(f"# ({title}; cold-cache serialised launches: compare shares, not absolute times, with bench.py)")
    print("# the measured step starts at the last k_meta")
    for k, us in out:
        print(f"{us:9.2f} us  {k}")
    tot = {}
    for k, us in step:
        name = re.sub(r"\(.*", "", k).replace("void ", "").replace("predtop::", "")
        name = re.sub(r"\(anonymous namespace\)::|unnamed>::", "", name)
        tot[name] = tot.get(name, 0.0) + us
    s = sum(tot.values())
    print(f"# measured step: {len(step)} launches, {s:.1f} us")
    for k, us in sorted(tot.items(), key=lambda x: -x[1]):
        print(f"#   {k[:44]:44s} {us:9.1f} us  {100 * us / s:5.1f} %")


if __name__ == "__main__":
    main()
