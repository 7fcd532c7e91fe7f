"""Compare the two fused layer-tail kernels (layer.cu v1 vs layer2.cu v2) on
the node embeddings after each layer: where (tile, row, column) do they differ?
Usage: python tools/tail_check.py [graphs]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ipps_acharyas25_b200 import build, predtop as pt, synth  # noqa: E402


def main():
    G = int(sys.argv[1]) if len(sys.argv) > 1 else 24
    build.build_library()
    cfg = dict(synth.MODEL_CONFIGS["gpt"])
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    model = pt.Model(cfg, blob)
    b = synth.stage_batch("gpt", G)
    dag = pt.Dag(pt.DeviceBatch.from_host(b))
    thr = float(sys.argv[2]) if len(sys.argv) > 2 else 1e-2
    import oracle
    taps = [oracle.forward(cfg, blob, *b.graph(g), taps=True)[2] for g in range(min(G, 4))]
    for layer in [0, 1, 0, 1, 1, 1, 2, 3]:
        os.environ["PREDTOP_TAIL_V1"] = "1"
        x1 = model.node_embeddings(dag, layer).cpu().numpy()
        os.environ["PREDTOP_TAIL_V1"] = "0"
        x2 = model.node_embeddings(dag, layer).cpu().numpy()
        torch.cuda.synchronize()
        d = np.abs(x1 - x2)
        rows = d.max(axis=1)
        bad = np.nonzero(rows > thr)[0]
        print(f"layer {layer}: M={x1.shape[0]} max abs diff {d.max():.3e}, median row max {np.median(rows):.3e}, "
              f"rows > {thr}: {bad.size}")
        if d.max() < 1e-2:
            continue
        want = np.concatenate([t[layer + 1] for t in taps])
        n = want.shape[0]
        print(f"  vs oracle (first {len(taps)} graphs): v1 {np.abs(x1[:n] - want).max():.3e} v2 {np.abs(x2[:n] - want).max():.3e}")
        if bad.size:
            tiles = sorted(set((bad // 128).tolist()))
            print("  tiles", tiles[:20], " rows%128", sorted(set((bad % 128).tolist()))[:40])
            cols = np.nonzero(d[bad].max(axis=0) > 1e-2)[0]
            print("  cols", cols[:64].tolist())
            r = bad[0]
            c = int(np.argmax(d[r]))
            print("  row", r, "col", c, "v1", x1[r, c], "v2", x2[r, c])
            worst = np.argsort(rows)[::-1][:6]
            for w in worst:
                cc = np.nonzero(d[w] > 1e-2)[0]
                print(f"  worst row {w} (tile {w // 128}, r {w % 128}) max {rows[w]:.3e} cols>1e-2 {cc.tolist()[:40]}")
            print("  diff histogram rows:", np.histogram(np.log10(rows + 1e-12), bins=[-12, -7, -6, -5, -4, -3, -2, 0])[0])


if __name__ == "__main__":
    main()
