"""CPU study of where the GPU path's fp16 roundings cost accuracy.

Emulates the GPU numerics in torch float32 with fp16 rounding at the points
the kernels round (x16 for GEMM inputs, q/k/v, P, attention output, h16,
ReLU output), compares the stage latency with the fp64 oracle, and reports
the error with each rounding point disabled in turn.
Usage: python tools/precision_study.py [num_graphs]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
from paper_conf_ipps_acharyas25_b200 import synth  # noqa: E402

POINTS = ["x16", "qkv", "P", "att", "h16", "relu"]
EX16 = os.environ.get("EX16") == "1"


def r16(t, on):
    return t.half().float() if on else t


def forward(cfg, w, n, s, d, f, off=()):
    on = {p: p not in off for p in POINTS}
    D, H, L = cfg["d_model"], cfg["num_heads"], cfg["num_layers"]
    dh = D // H
    T = lambda a: torch.from_numpy(np.asarray(a, np.float32))
    dep = oracle.depth(n, s, d)
    M = torch.from_numpy(oracle.bits_to_dense(oracle.mask(n, oracle.reach(n, s, d)), n))
    x = torch.from_numpy(oracle.embed(cfg, synth.pack_weights(cfg, w), n, f, dep)).float()
    for l in range(L):
        g = lambda k: T(w[f"L{l}.{k}"])
        qkv = r16(r16(x, on["x16"]) @ g("W_qkv").T + g("b_qkv"), on["qkv"])
        q, k, v = qkv[:, :D], qkv[:, D:2 * D], qkv[:, 2 * D:]
        att = torch.empty(n, D)
        for hh in range(H):
            sl = slice(hh * dh, (hh + 1) * dh)
            sc = (q[:, sl] @ k[:, sl].T) / np.sqrt(dh)
            sc = sc.masked_fill(~M, float("-inf"))
            if EX16:
                # kernel v9 candidate: exp2 on fp16 arguments (ex2.approx.f16x2):
                # m = diagonal score unless the row max exceeds it by > 8
                l2 = sc * np.log2(np.e)
                mx = l2.max(1, keepdim=True).values
                dg = torch.diagonal(l2).unsqueeze(1)
                m = torch.where(mx > dg + 8, mx, dg)
                p16 = torch.exp2((l2 - m).half().float()).half().float()
            else:
                p = torch.exp(sc - sc.max(1, keepdim=True).values)
                p16 = r16(p, on["P"])
            att[:, sl] = (p16 @ v[:, sl]) / p16.sum(1, keepdim=True)
        att = r16(att, on["att"])
        z = x + att @ g("W_o").T + g("b_o")
        h = torch.nn.functional.layer_norm(z, (D,), g("ln1_g"), g("ln1_b"), cfg["ln_eps"])
        u = r16(torch.relu(r16(h, on["h16"]) @ g("W_1").T + g("b_1")), on["relu"])
        z2 = h + u @ g("W_2").T + g("b_2")
        x = torch.nn.functional.layer_norm(z2, (D,), g("ln2_g"), g("ln2_b"), cfg["ln_eps"])
    gp = x.double().sum(0)
    Td = lambda a: torch.from_numpy(np.asarray(a, np.float64))
    z = torch.relu(Td(w["H_1"]) @ gp + Td(w["c_1"]))
    z = torch.relu(Td(w["H_2"]) @ z + Td(w["c_2"]))
    return float(Td(w["w_o"]) @ z + Td(w["c_o"]))


def main():
    G = int(sys.argv[1]) if len(sys.argv) > 1 else 24
    cfg = synth.MODEL_CONFIGS["gpt"]
    w = synth.model_weights(cfg)
    blob = synth.pack_weights(cfg, w)
    b = synth.stage_batch("gpt", G)
    ref = oracle.forward_batch(cfg, blob, b)
    rows = {}
    for off in [(), *[(p,) for p in POINTS], tuple(POINTS)]:
        y = np.asarray([forward(cfg, w, *b.graph(g), off=off) for g in range(G)])
        e = np.abs(y - ref) / np.abs(ref)
        rows[off] = e
        print(f"off={','.join(off) or 'none':32s} max {e.max():.3e} (g{e.argmax()}) median {np.median(e):.3e} rms {np.sqrt((e**2).mean()):.3e}")
    print("y of worst graph:", ref[rows[()].argmax()])


if __name__ == "__main__":
    main()
