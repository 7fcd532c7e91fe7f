"""Pins of the oracle's DAG-Transformer steps.

Library special cases (torch float64 on CPU, outside the oracle tree):
  * Eqn 1 masked attention == F.scaled_dot_product_attention with
    a boolean mask built from brute-force reachability;
  * the layer (Fig. 4, reading R6) == nn.TransformerEncoderLayer(post-LN, ReLU)
    of [34] with the same weights and src_mask = not-allowed;
  * the readout / head (Eqn 2 P:174) == sum + nn.Sequential MLP.
Closed forms: Table I one-hot positions and ln(1+dim) values (P:147-157,
P:167); PE(depth=0) = [0,1,0,1,...]; frequencies form a geometric progression
from 1 to 1/10000 ([34]).  Invariants: antichain -> O = V exactly; disjoint
union block independence; relabelling invariance (DAGPE/DAGRA depend only on
the graph).
"""
import math

import numpy as np
import pytest
import torch
import torch.nn.functional as Fn

from paper_conf_ipps_acharyas25_b200 import synth


def _cfg(name="tiny", **kw):
    c = dict(synth.MODEL_CONFIGS[name])
    c.update(kw)
    return c


def _blob(cfg):
    w = synth.model_weights(cfg)
    return w, synth.pack_weights(cfg, w)


def _dense(oracle_mod, B, n):
    return oracle_mod.bits_to_dense(B, n)


def _graph(n=37, p=0.08, seed=5):
    rng = synth.CounterRng(seed, n)
    s, d = synth.random_dag(n, p, rng)
    return n, s, d, synth._rand_feats(n, rng)


def test_blob_length(oracle_mod):
    for name in synth.MODEL_CONFIGS:
        cfg = synth.MODEL_CONFIGS[name]
        assert oracle_mod.blob_floats(cfg) == len(synth.pack_weights(cfg, synth.model_weights(cfg)))


def test_features_closed_forms(oracle_mod):
    f = np.zeros(3, synth.FEAT_DTYPE)
    f[0] = (5, 2, 3, (0, 1, 4294967295, 7))
    f[1] = (63, 7, 0, (1, 1, 1, 1))
    f[2] = (64, 8, 4, (0, 0, 0, 0))  # out of vocabulary -> zero one-hots
    X = oracle_mod.features(3, f)
    assert X.shape == (3, 80)
    # row 0
    assert X[0, 5] == 1.0 and X[0, :64].sum() == 1.0
    assert X[0, 64] == 0.0 and X[0, 65] == pytest.approx(math.log(2.0), abs=1e-15)
    assert X[0, 66] == pytest.approx(32 * math.log(2.0), rel=1e-15)
    assert X[0, 67] == pytest.approx(3 * math.log(2.0), rel=1e-15)
    assert X[0, 68 + 2] == 1.0 and X[0, 68:76].sum() == 1.0
    assert X[0, 76 + 3] == 1.0 and X[0, 76:80].sum() == 1.0
    # row 1
    assert X[1, 63] == 1.0 and X[1, 75] == 1.0 and X[1, 76] == 1.0
    # row 2: nothing but zeros
    assert not X[2].any()


def test_embedding_linear_part_and_pe(oracle_mod):
    cfg = _cfg("paper")
    w, blob = _blob(cfg)
    n, s, d, f = _graph(20)
    d_model = cfg["d_model"]
    zero = np.zeros(n, np.int32)
    x0 = oracle_mod.embed(cfg, blob, n, f, zero)
    feats = torch.from_numpy(oracle_mod.features(n, f))
    lin = Fn.linear(feats, torch.from_numpy(w["W_in"]).double(), torch.from_numpy(w["b_in"]).double())
    pe0 = np.tile([0.0, 1.0], d_model // 2)  # PE(0) = [sin 0, cos 0, ...]
    np.testing.assert_allclose(x0, lin.numpy() + pe0, rtol=0, atol=1e-12)
    # PE alone: embed(depth) - embed(0)
    depths = np.arange(n, dtype=np.int32) * 37
    pe = oracle_mod.embed(cfg, blob, n, f, depths) - lin.numpy()
    np.testing.assert_allclose(pe[:, 0], np.sin(depths), atol=1e-12)          # w_0 = 1
    np.testing.assert_allclose(pe[:, 1], np.cos(depths), atol=1e-12)
    np.testing.assert_allclose(pe[:, 0::2] ** 2 + pe[:, 1::2] ** 2, 1.0, atol=1e-12)
    # frequency of pair i from depth 1: geometric progression, ratio 10000^(-2/d),
    # reaching 1/10000 at i = d/2 ([34]: wavelengths 2pi .. 10000*2pi)
    one = oracle_mod.embed(cfg, blob, 1, f[:1], np.ones(1, np.int32)) - lin.numpy()[:1]
    w_i = np.arctan2(one[0, 0::2], one[0, 1::2])
    ratio = w_i[1:] / w_i[:-1]
    np.testing.assert_allclose(ratio, ratio[0], rtol=1e-9)
    assert w_i[0] == pytest.approx(1.0, abs=1e-12)
    assert w_i[0] * ratio[0] ** (d_model // 2) == pytest.approx(1e-4, rel=1e-7)


def _torch_attention(cfg, w, layer, x, allowed):
    d, H = cfg["d_model"], cfg["num_heads"]
    dh = d // H
    qkv = Fn.linear(torch.from_numpy(x), torch.from_numpy(w[f"L{layer}.W_qkv"]).double(),
                    torch.from_numpy(w[f"L{layer}.b_qkv"]).double())
    q, k, v = qkv[:, :d], qkv[:, d:2 * d], qkv[:, 2 * d:]
    n = x.shape[0]
    q = q.reshape(n, H, dh).transpose(0, 1)
    k = k.reshape(n, H, dh).transpose(0, 1)
    v = v.reshape(n, H, dh).transpose(0, 1)
    o = Fn.scaled_dot_product_attention(q, k, v, attn_mask=torch.from_numpy(allowed))
    return o.transpose(0, 1).reshape(n, d).numpy(), v.transpose(0, 1).reshape(n, d).numpy()


@pytest.mark.parametrize("shape", ["chain", "random", "antichain"])
def test_attention_vs_sdpa(oracle_mod, shape):
    cfg = _cfg("paper")
    w, blob = _blob(cfg)
    n = 45
    if shape == "chain":
        s, d = synth.chain(n)
    elif shape == "antichain":
        s, d = np.zeros(0, np.int32), np.zeros(0, np.int32)
    else:
        s, d = synth.random_dag(n, 0.05, synth.CounterRng(1, 2))
    M = oracle_mod.mask(n, oracle_mod.reach(n, s, d))
    allowed = _dense(oracle_mod, M, n)
    if shape == "chain":
        assert allowed.all()  # M all-ones: plain dense attention
    x = synth.CounterRng(8, 8).uniform_array(n * cfg["d_model"]).reshape(n, -1) * 2 - 1
    got = oracle_mod.attention(cfg, blob, 0, n, M, x)
    want, v = _torch_attention(cfg, w, 0, x, allowed)
    np.testing.assert_allclose(got, want, rtol=1e-12, atol=1e-12)
    if shape == "antichain":  # M = I: softmax over one element -> O = V
        np.testing.assert_allclose(got, v, rtol=0, atol=1e-14)


@pytest.mark.parametrize("name", ["tiny", "paper", "gpt"])
def test_layer_vs_torch_encoder_layer(oracle_mod, name):
    cfg = _cfg(name)
    w, blob = _blob(cfg)
    d, H, dff = cfg["d_model"], cfg["num_heads"], cfg["d_ff"]
    n, s, dd, f = _graph(70, 0.04, seed=3)
    M = oracle_mod.mask(n, oracle_mod.reach(n, s, dd))
    allowed = _dense(oracle_mod, M, n)
    x = synth.CounterRng(4, 4).uniform_array(n * d).reshape(n, d) * 4 - 2
    got = oracle_mod.layer(cfg, blob, 0, n, M, x)
    enc = torch.nn.TransformerEncoderLayer(d, H, dff, dropout=0.0, activation="relu",
                                           layer_norm_eps=cfg["ln_eps"], batch_first=True,
                                           norm_first=False, dtype=torch.float64)
    T = lambda a: torch.from_numpy(np.asarray(a)).double()
    with torch.no_grad():
        enc.self_attn.in_proj_weight.copy_(T(w["L0.W_qkv"]))
        enc.self_attn.in_proj_bias.copy_(T(w["L0.b_qkv"]))
        enc.self_attn.out_proj.weight.copy_(T(w["L0.W_o"]))
        enc.self_attn.out_proj.bias.copy_(T(w["L0.b_o"]))
        enc.linear1.weight.copy_(T(w["L0.W_1"]))
        enc.linear1.bias.copy_(T(w["L0.b_1"]))
        enc.linear2.weight.copy_(T(w["L0.W_2"]))
        enc.linear2.bias.copy_(T(w["L0.b_2"]))
        enc.norm1.weight.copy_(T(w["L0.ln1_g"]))
        enc.norm1.bias.copy_(T(w["L0.ln1_b"]))
        enc.norm2.weight.copy_(T(w["L0.ln2_g"]))
        enc.norm2.bias.copy_(T(w["L0.ln2_b"]))
        enc.train()  # the reference math path, no fused fast path (dropout=0 anyway)
        want = enc(T(x)[None], src_mask=torch.from_numpy(~allowed))[0].numpy()
    np.testing.assert_allclose(got, want, rtol=1e-10, atol=1e-10)


def _torch_head(cfg, w, g):
    T = lambda a: torch.from_numpy(np.asarray(a)).double()
    z = torch.relu(Fn.linear(T(g), T(w["H_1"]), T(w["c_1"])))
    z = torch.relu(Fn.linear(z, T(w["H_2"]), T(w["c_2"])))
    return float(Fn.linear(z, T(w["w_o"]), T(w["c_o"]))[0])


@pytest.mark.parametrize("pool", [0, 1])
def test_readout_vs_torch(oracle_mod, pool):
    cfg = _cfg("gpt", pool=pool)
    w, blob = _blob(cfg)
    n = 33
    x = synth.CounterRng(2, 2).uniform_array(n * cfg["d_model"]).reshape(n, -1) * 2 - 1
    g = x.sum(0) / (n if pool == 1 else 1)
    assert oracle_mod.readout(cfg, blob, n, x) == pytest.approx(_torch_head(cfg, w, g), rel=1e-12)


def test_block_independence_and_pool_additivity(oracle_mod):
    """Disjoint union A (+) B: node embeddings equal those of A and B computed
    separately, bit-exactly (masked terms are exact zeros, Eqn 1), and the
    pooled vector is the sum of the two pools (Eqn 2)."""
    cfg = _cfg("paper")
    w, blob = _blob(cfg)
    nA, sA, dA, fA = _graph(23, 0.1, seed=1)
    nB, sB, dB, fB = _graph(17, 0.15, seed=2)
    n = nA + nB
    s = np.concatenate([sA, sB + nA]).astype(np.int32)
    d = np.concatenate([dA, dB + nA]).astype(np.int32)
    f = np.concatenate([fA, fB])
    _, yU, tU = oracle_mod.forward(cfg, blob, n, s, d, f, taps=True)
    _, yA, tA = oracle_mod.forward(cfg, blob, nA, sA, dA, fA, taps=True)
    _, yB, tB = oracle_mod.forward(cfg, blob, nB, sB, dB, fB, taps=True)
    np.testing.assert_array_equal(tU[:, :nA], tA)
    np.testing.assert_array_equal(tU[:, nA:], tB)
    g = tA[-1].sum(0) + tB[-1].sum(0)
    assert yU == pytest.approx(_torch_head(cfg, w, g), rel=1e-12)


@pytest.mark.parametrize("name", ["tiny", "gpt"])
def test_relabelling_invariance(oracle_mod, name):
    cfg = _cfg(name)
    _, blob = _blob(cfg)
    b = synth.stage_batch("gpt", 1) if name == "gpt" else synth.tiny_batch()
    n, s, d, f = b.graph(0)
    perm = synth.CounterRng(77, 1).permutation(n)
    s2, d2, f2 = synth.relabel(n, s, d, f, perm)
    st1, y1, t1 = oracle_mod.forward(cfg, blob, n, s, d, f, taps=True)
    st2, y2, t2 = oracle_mod.forward(cfg, blob, n, s2, d2, f2, taps=True)
    assert st1 == st2 == 0
    assert y2 == pytest.approx(y1, rel=1e-12)
    np.testing.assert_allclose(t2[:, perm], t1, rtol=1e-11, atol=1e-11)


def test_full_forward_composes_steps(oracle_mod):
    """orc_forward == embed -> layers -> readout composed from the pinned
    steps (catches a wiring mistake in the composition)."""
    cfg = _cfg("paper")
    w, blob = _blob(cfg)
    n, s, d, f = _graph(50, 0.06, seed=9)
    dep = oracle_mod.depth(n, s, d)
    M = oracle_mod.mask(n, oracle_mod.reach(n, s, d))
    x = oracle_mod.embed(cfg, blob, n, f, dep)
    for l in range(cfg["num_layers"]):
        x = oracle_mod.layer(cfg, blob, l, n, M, x)
    st, y, taps = oracle_mod.forward(cfg, blob, n, s, d, f, taps=True)
    assert st == 0
    np.testing.assert_array_equal(taps[-1], x)
    assert y == oracle_mod.readout(cfg, blob, n, x)


def test_invalid_graph_gives_nan(oracle_mod):
    cfg = _cfg("tiny")
    _, blob = _blob(cfg)
    f = np.zeros(3, synth.FEAT_DTYPE)
    st, y, _ = oracle_mod.forward(cfg, blob, 3, np.array([0, 1, 2]), np.array([1, 2, 0]), f)
    assert st == oracle_mod.CYCLE and math.isnan(y)


def test_row_block_evaluation_is_the_same_layer(oracle_mod):
    """oracle.layer_rows / forward_rows (the 16k path: one graph's layers
    evaluated row block by row block on several threads) compose the same
    orc_qkv_rows / orc_attention_rows / orc_layer_post_rows that orc_layer
    is built from, so they reproduce orc_layer / orc_forward bit for bit, for
    any row subset and any thread count."""
    from paper_conf_ipps_acharyas25_b200 import synth
    cfg = synth.MODEL_CONFIGS["paper"]
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    b = synth.stage_batch("gpt", 2, first_graph=9)
    for g in range(2):
        n, s, d, f = b.graph(g)
        st, y, taps = oracle_mod.forward(cfg, blob, n, s, d, f, taps=True)
        st2, y2, taps2 = oracle_mod.forward_rows(cfg, blob, n, s, d, f, threads=3, taps=True)
        assert st == st2 == 0 and y == y2
        np.testing.assert_array_equal(taps, taps2)
        M = oracle_mod.mask(n, oracle_mod.reach(n, s, d))
        rows = [0, 1, 2, 40, 41, n - 1]
        np.testing.assert_array_equal(oracle_mod.layer_rows(cfg, blob, 2, n, M, taps[2], rows=rows, threads=2),
                                      oracle_mod.layer(cfg, blob, 2, n, M, taps[2])[rows])


@pytest.mark.parametrize("pool", [0, 1])
def test_head_condition_bounds_bias_free_output(oracle_mod, pool):
    """oracle.head_condition (reading R22) is the absolute sum of the terms of
    y - c_o = w_o . h2: it bounds |y - c_o| (triangle inequality), and equals
    it when every w_o,i >= 0 (h2 >= 0 after the ReLU), on the oracle readout."""
    cfg = _cfg("gpt", pool=pool)
    w, blob = _blob(cfg)
    n = 29
    x = synth.CounterRng(3, 3).uniform_array(n * cfg["d_model"]).reshape(n, -1) * 2 - 1
    c_o = float(w["c_o"][0])
    y = oracle_mod.readout(cfg, blob, n, x)
    assert oracle_mod.head_condition(cfg, blob, n, x) >= abs(y - c_o) * (1 - 1e-12)
    w2 = dict(w)
    w2["w_o"] = np.abs(w["w_o"])
    blob2 = synth.pack_weights(cfg, w2)
    y2 = oracle_mod.readout(cfg, blob2, n, x)
    assert oracle_mod.head_condition(cfg, blob2, n, x) == pytest.approx(y2 - c_o, rel=1e-12)
