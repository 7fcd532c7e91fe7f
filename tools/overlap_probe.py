"""Probe: does splitting the GPT batch into two halves on two streams (so the
MUFU-bound attention of one half can co-run with the tensor/TMA-bound layer
tail of the other) beat one stream?  Times build + forward per step with
CUDA graphs.  Usage: python tools/overlap_probe.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_acharyas25_b200 import predtop as pt, synth  # noqa: E402


def main():
    cfg = synth.MODEL_CONFIGS["gpt"]
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    model = pt.Model(cfg, blob)
    host = synth.stage_batch("gpt", 1024)
    halves = [host.subset(range(0, 512)), host.subset(range(512, 1024))]
    full = pt.DeviceBatch.from_host(host)
    dag = pt.Dag(full, no_sync=True)
    ws = model.forward_workspace(dag)
    lat = torch.empty(1024, device="cuda")
    hb = [pt.DeviceBatch.from_host(h) for h in halves]
    hd = [pt.Dag(b, no_sync=True) for b in hb]
    hws = [model.forward_workspace(d) for d in hd]
    hl = [torch.empty(512, device="cuda") for _ in range(2)]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    main_s = torch.cuda.current_stream()

    def one():
        dag.rebuild()
        model.forward(dag, ws, lat)

    def two():
        cur = torch.cuda.current_stream()
        for k in range(2):
            streams[k].wait_stream(cur)
            with torch.cuda.stream(streams[k]):
                hd[k].rebuild()
                model.forward(hd[k], hws[k], hl[k])
        for k in range(2):
            cur.wait_stream(streams[k])

    def graph(fn):
        side = torch.cuda.Stream()
        side.wait_stream(main_s)
        with torch.cuda.stream(side):
            fn()
        main_s.wait_stream(side)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            fn()
        torch.cuda.synchronize()
        return g

    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for name, fn in [("one stream", one), ("two halves, two streams", two)]:
        g = graph(fn)
        for _ in range(3):
            g.replay()
        ts = []
        for _ in range(20):
            flush.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            g.replay()
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        ts.sort()
        print(f"{name}: median {ts[len(ts) // 2]:.3f} ms  -> {1024 / ts[len(ts) // 2] * 1e3:.0f} graphs/s")
    torch.cuda.synchronize()
    print("max |diff| halves vs full:", (torch.cat(hl) - lat).abs().max().item())


if __name__ == "__main__":
    main()
