"""Pins of the oracle's training functions.

* orc_grad (the reverse of every forward step) against
  - central finite differences of the oracle forward itself, with exactly
    representable weight perturbations (h = 2^-12 on float32 weights >= 2^-12
    in magnitude, so w +- h is exact and only the O(h^2) truncation remains);
  - torch float64 autograd of the same model assembled from library modules
    (nn.TransformerEncoderLayer post-LN/ReLU with the reachability mask, Linear
    embedding + the oracle's own PE as a constant, sum pool, Linear/ReLU head)
    under nn.L1Loss over a batch (Eqn 3 MAE).
* adam_step against torch.optim.Adam (PyTorch's Adam, defaults).
* cosine_lr against torch's CosineAnnealingLR (1e-3 -> 0).
"""
import numpy as np
import pytest
import torch

from paper_conf_ipps_acharyas25_b200 import synth

TRAIN_CFG = dict(num_layers=2, d_model=16, num_heads=2, d_ff=32, pool=0, ln_eps=1e-5,
                 head_scale=0.5, out_bias=1.0, seed=120)


def _graph(n, p, seed):
    rng = synth.CounterRng(seed, n)
    s, d = synth.random_dag(n, p, rng)
    return n, s, d, synth._rand_feats(n, rng)


def test_grad_vs_finite_differences(oracle_mod):
    cfg = TRAIN_CFG
    w = synth.model_weights(cfg)
    blob = synth.pack_weights(cfg, w).astype(np.float32)
    n, s, d, f = _graph(11, 0.2, 3)
    y0, g = oracle_mod.grad(cfg, blob, n, s, d, f)
    assert y0 == pytest.approx(oracle_mod.forward(cfg, blob, n, s, d, f)[1], rel=1e-14)
    h = 2.0 ** -12
    # two sampled entries of every tensor, each with |w| >= 2^-12 (exact w +- h)
    rng = np.random.default_rng(7)
    off = 0
    checked = 0
    for name, shape in synth.weight_shapes(cfg):
        size = int(np.prod(shape))
        cand = [off + i for i in range(size) if abs(blob[off + i]) >= 2.0 ** -12]
        for idx in rng.choice(cand, size=min(2, len(cand)), replace=False):
            bp = blob.copy()
            bm = blob.copy()
            bp[idx] += np.float32(h)
            bm[idx] -= np.float32(h)
            assert float(bp[idx]) - float(blob[idx]) == h and float(blob[idx]) - float(bm[idx]) == h
            fd = (oracle_mod.forward(cfg, bp, n, s, d, f)[1] - oracle_mod.forward(cfg, bm, n, s, d, f)[1]) / (2 * h)
            assert abs(fd - g[idx]) <= 1e-6 + 1e-5 * abs(g[idx]), (name, idx, fd, g[idx])
            checked += 1
        off += size
    assert checked >= 2 * len(synth.weight_shapes(cfg)) - 2


class _TorchModel(torch.nn.Module):
    """The DAG-Transformer of DESIGN readings R1-R11 from torch library modules."""

    def __init__(self, cfg, w):
        super().__init__()
        d, H, dff, L = cfg["d_model"], cfg["num_heads"], cfg["d_ff"], cfg["num_layers"]
        T = lambda a: torch.nn.Parameter(torch.from_numpy(np.asarray(a, np.float64)).clone())
        self.W_in, self.b_in = T(w["W_in"]), T(w["b_in"])
        self.layers = torch.nn.ModuleList()
        for l in range(L):
            enc = torch.nn.TransformerEncoderLayer(d, H, dff, dropout=0.0, activation="relu",
                                                   layer_norm_eps=cfg["ln_eps"], batch_first=True,
                                                   norm_first=False, dtype=torch.float64)
            with torch.no_grad():
                for tgt, key in [(enc.self_attn.in_proj_weight, "W_qkv"), (enc.self_attn.in_proj_bias, "b_qkv"),
                                 (enc.self_attn.out_proj.weight, "W_o"), (enc.self_attn.out_proj.bias, "b_o"),
                                 (enc.linear1.weight, "W_1"), (enc.linear1.bias, "b_1"),
                                 (enc.linear2.weight, "W_2"), (enc.linear2.bias, "b_2"),
                                 (enc.norm1.weight, "ln1_g"), (enc.norm1.bias, "ln1_b"),
                                 (enc.norm2.weight, "ln2_g"), (enc.norm2.bias, "ln2_b")]:
                    tgt.copy_(torch.from_numpy(np.asarray(w[f"L{l}.{key}"], np.float64)))
            enc.train()
            self.layers.append(enc)
        self.H1, self.c1, self.H2, self.c2 = T(w["H_1"]), T(w["c_1"]), T(w["H_2"]), T(w["c_2"])
        self.w_o, self.c_o = T(w["w_o"]), T(w["c_o"])

    def forward(self, F, pe, not_allowed):
        x = F @ self.W_in.T + self.b_in + pe
        for enc in self.layers:
            x = enc(x[None], src_mask=not_allowed)[0]
        g = x.sum(0)
        z = torch.relu(g @ self.H1.T + self.c1)
        z = torch.relu(z @ self.H2.T + self.c2)
        return (z @ self.w_o.T + self.c_o)[0]

    def grads(self, cfg):
        """Gradients in the weight-blob order of synth.weight_shapes."""
        by = {"W_in": self.W_in, "b_in": self.b_in, "H_1": self.H1, "c_1": self.c1, "H_2": self.H2,
              "c_2": self.c2, "w_o": self.w_o, "c_o": self.c_o}
        for l, enc in enumerate(self.layers):
            for key, p in [("W_qkv", enc.self_attn.in_proj_weight), ("b_qkv", enc.self_attn.in_proj_bias),
                           ("W_o", enc.self_attn.out_proj.weight), ("b_o", enc.self_attn.out_proj.bias),
                           ("W_1", enc.linear1.weight), ("b_1", enc.linear1.bias),
                           ("W_2", enc.linear2.weight), ("b_2", enc.linear2.bias),
                           ("ln1_g", enc.norm1.weight), ("ln1_b", enc.norm1.bias),
                           ("ln2_g", enc.norm2.weight), ("ln2_b", enc.norm2.bias)]:
                by[f"L{l}.{key}"] = p
        return np.concatenate([by[name].grad.numpy().ravel() for name, _ in synth.weight_shapes(cfg)])


@pytest.mark.parametrize("name", ["train", "tiny"])
def test_mae_grad_vs_torch_autograd(oracle_mod, name):
    cfg = TRAIN_CFG if name == "train" else dict(synth.MODEL_CONFIGS["tiny"])
    w = synth.model_weights(cfg)
    blob = synth.pack_weights(cfg, w)
    graphs = [_graph(9, 0.25, 1), _graph(14, 0.15, 2), _graph(6, 0.4, 4)]
    batch = synth.pack_graphs(graphs)
    y_true = np.array([0.5, 9.0, -1.0])
    loss, g, y_hat = oracle_mod.mae_grad(cfg, blob, batch, y_true, threads=1)
    model = _TorchModel(cfg, w)
    preds = []
    for (n, s, d, f) in graphs:
        F = torch.from_numpy(oracle_mod.features(n, f))
        dep = oracle_mod.depth(n, s, d)
        x0 = oracle_mod.embed(cfg, blob, n, f, dep)
        pe = torch.from_numpy(x0 - (F.numpy() @ np.asarray(w["W_in"], np.float64).T + w["b_in"]))
        allowed = oracle_mod.bits_to_dense(oracle_mod.mask(n, oracle_mod.reach(n, s, d)), n)
        preds.append(model(F, pe, torch.from_numpy(~allowed)))
    yt = torch.stack(preds)
    L = torch.nn.L1Loss()(yt, torch.from_numpy(y_true))
    L.backward()
    np.testing.assert_allclose(y_hat, yt.detach().numpy(), rtol=1e-11)
    assert loss == pytest.approx(float(L.detach()), rel=1e-12)
    want = model.grads(cfg)
    np.testing.assert_allclose(g, want, rtol=1e-8, atol=1e-11 * np.abs(want).max())


def test_adam_vs_torch():
    rng = np.random.default_rng(3)
    p0 = rng.standard_normal(50)
    grads = [rng.standard_normal(50) for _ in range(6)]
    import oracle
    p, m, v = p0.copy(), np.zeros(50), np.zeros(50)
    for t, g in enumerate(grads, start=1):
        p, m, v = oracle.adam_step(p, g, m, v, t, lr=1e-3 * (1 + t))
    tp = torch.nn.Parameter(torch.from_numpy(p0.copy()))
    opt = torch.optim.Adam([tp], lr=1e-3)
    for t, g in enumerate(grads, start=1):
        for grp in opt.param_groups:
            grp["lr"] = 1e-3 * (1 + t)
        tp.grad = torch.from_numpy(g)
        opt.step()
    np.testing.assert_allclose(p, tp.detach().numpy(), rtol=1e-13, atol=1e-15)


def test_cosine_lr_vs_torch():
    import oracle
    E = 37
    tp = torch.nn.Parameter(torch.zeros(1))
    opt = torch.optim.SGD([tp], lr=1e-3)
    sch = torch.optim.lr_scheduler.CosineAnnealingLR(opt, T_max=E - 1, eta_min=0.0)
    for e in range(E):
        assert oracle.cosine_lr(e, E, 1e-3) == pytest.approx(opt.param_groups[0]["lr"], rel=1e-12, abs=1e-18)
        opt.step()
        sch.step()
    assert oracle.cosine_lr(0, E) == 1e-3 and abs(oracle.cosine_lr(E - 1, E)) < 1e-18
