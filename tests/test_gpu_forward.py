"""GPU parity of the DAG-Transformer forward (predtop_stage_forward) against the
CPU fp64 oracle, per graph relative error <= 2e-3 (BASELINE.json north star),
plus layer-wise taps (localisation), determinism and shard invariance
(per-graph outputs bit-identical whatever the batch composition)."""
import numpy as np
import pytest
import torch

from paper_conf_ipps_acharyas25_b200 import synth

pytestmark = pytest.mark.gpu
TOL = 2e-3


@pytest.fixture(scope="module")
def pt():
    from paper_conf_ipps_acharyas25_b200 import build, predtop
    build.build_library()
    assert torch.cuda.is_available()
    return predtop


def _model(pt, name, **kw):
    cfg = dict(synth.MODEL_CONFIGS[name])
    cfg.update(kw)
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    return cfg, blob, pt.Model(cfg, blob)


def _gpu_latency(pt, model, batch):
    dag = pt.Dag(pt.DeviceBatch.from_host(batch))
    assert dag.status == pt.OK
    y = model.forward(dag)
    torch.cuda.synchronize()
    return y.cpu().numpy().astype(np.float64), dag


def _rel(a, b):
    return np.abs(a - b) / np.abs(b)


@pytest.mark.parametrize("name, batch_fn", [
    ("tiny", lambda: synth.tiny_batch()),
    ("paper", lambda: synth.stage_batch("gpt", 12, seed=11)),
    ("gpt", lambda: synth.stage_batch("gpt", 24)),
    ("moe", lambda: synth.stage_batch("moe", 3)),
])
def test_latency_parity(pt, oracle_mod, name, batch_fn):
    cfg, blob, model = _model(pt, name)
    batch = batch_fn()
    y, _ = _gpu_latency(pt, model, batch)
    want = oracle_mod.forward_batch(cfg, blob, batch)
    err = _rel(y, want)
    print(f"{name}: max rel err {err.max():.3e} median {np.median(err):.3e}")
    assert np.isfinite(y).all()
    assert err.max() <= TOL


@pytest.mark.parametrize("name, batch_fn", [
    ("paper", lambda: synth.stage_batch("gpt", 12, seed=11)),
    ("gpt", lambda: synth.stage_batch("gpt", 24)),
    ("gpt", lambda: synth.tiny_batch()),
])
def test_latency_parity_tcgen05_attention(pt, oracle_mod, name, batch_fn, monkeypatch):
    """The opt-in tcgen05/TMEM attention kernel (attention_tc.cu, d_h = 16)."""
    monkeypatch.setenv("PREDTOP_ATTN_TC", "1")
    cfg, blob, model = _model(pt, name)
    batch = batch_fn()
    y, _ = _gpu_latency(pt, model, batch)
    want = oracle_mod.forward_batch(cfg, blob, batch)
    err = _rel(y, want)
    print(f"{name} (tcgen05 attention): max rel err {err.max():.3e}")
    assert np.isfinite(y).all()
    assert err.max() <= TOL


@pytest.mark.parametrize("name, batch_fn", [
    ("gpt", lambda: synth.stage_batch("gpt", 24)),
    ("gpt", lambda: synth.stage_batch("gpt", 5, seed=7)),
])
def test_latency_parity_tail_v1(pt, oracle_mod, name, batch_fn, monkeypatch):
    """The one-CTA-per-SM fused layer tail (layer.cu, PREDTOP_TAIL_V1=1) that
    the default two-CTA kernel (layer2.cu) replaced at d = 128."""
    monkeypatch.setenv("PREDTOP_TAIL_V1", "1")
    cfg, blob, model = _model(pt, name)
    batch = batch_fn()
    y, _ = _gpu_latency(pt, model, batch)
    want = oracle_mod.forward_batch(cfg, blob, batch)
    err = _rel(y, want)
    print(f"{name} (tail v1): max rel err {err.max():.3e}")
    assert np.isfinite(y).all()
    assert err.max() <= TOL


@pytest.mark.parametrize("name, batch_fn", [
    ("gpt", lambda: synth.stage_batch("gpt", 24)),
    ("gpt", lambda: synth.stage_batch("gpt", 7, first_graph=50)),
])
def test_latency_parity_tail_v3(pt, oracle_mod, name, batch_fn, monkeypatch):
    """The two-tiles-per-CTA fused layer tail (layer3.cu, PREDTOP_TAIL_V3=1);
    the second batch has an odd number of 128-row tiles (a half-empty pair)."""
    monkeypatch.setenv("PREDTOP_TAIL_V3", "1")
    cfg, blob, model = _model(pt, name)
    batch = batch_fn()
    y, _ = _gpu_latency(pt, model, batch)
    want = oracle_mod.forward_batch(cfg, blob, batch)
    err = _rel(y, want)
    print(f"{name} (tail v3): max rel err {err.max():.3e}")
    assert np.isfinite(y).all()
    assert err.max() <= TOL


@pytest.mark.parametrize("name, n", [("paper", 1700), ("moe", 800)])
def test_latency_parity_streaming_attention(pt, oracle_mod, name, n):
    """Graphs whose K/V do not fit shared memory (d_h = 16: N > 1536; d_h =
    32: N > 768) take the two-buffer TMA streaming path of the attention
    kernel; plus a small graph in the same batch."""
    rng = synth.CounterRng(7, n)
    s, d = synth.random_dag(n, 2.5 / n, rng)
    s2, d2 = synth.random_dag(90, 0.05, rng)
    batch = synth.pack_graphs([(n, s, d, synth._rand_feats(n, rng)), (90, s2, d2, synth._rand_feats(90, rng))])
    cfg, blob, model = _model(pt, name)
    y, _ = _gpu_latency(pt, model, batch)
    want = oracle_mod.forward_batch(cfg, blob, batch)
    err = _rel(y, want)
    print(f"{name} N={n}: max rel err {err.max():.3e}")
    assert np.isfinite(y).all()
    assert err.max() <= TOL


def test_mean_pool_and_relabelled(pt, oracle_mod):
    cfg, blob, model = _model(pt, "gpt", pool=1)
    b = synth.stage_batch("gpt", 4, first_graph=300)
    gs = []
    for g in range(b.num_graphs):
        n, s, d, f = b.graph(g)
        s2, d2, f2 = synth.relabel(n, s, d, f, synth.CounterRng(5, g).permutation(n))
        gs.append((n, s2, d2, f2))
    rb = synth.pack_graphs(gs)
    y, _ = _gpu_latency(pt, model, rb)
    want = oracle_mod.forward_batch(cfg, blob, rb)
    assert _rel(y, want).max() <= TOL


def test_layer_taps(pt, oracle_mod):
    """Embedding (fp32) and per-layer node embeddings against the oracle taps."""
    cfg, blob, model = _model(pt, "gpt")
    b = synth.stage_batch("gpt", 3, first_graph=50)
    dag = pt.Dag(pt.DeviceBatch.from_host(b))
    taps = [oracle_mod.forward(cfg, blob, *b.graph(g), taps=True)[2] for g in range(3)]
    for layer in range(-1, cfg["num_layers"]):
        x = model.node_embeddings(dag, layer).cpu().numpy()
        want = np.concatenate([t[layer + 1] for t in taps])
        err = np.abs(x - want).max()
        print(f"layer {layer}: max abs err {err:.3e}")
        assert err < (1e-4 if layer < 0 else 5e-2)


def test_determinism_and_shard_invariance(pt):
    cfg, blob, model = _model(pt, "gpt")
    full = synth.stage_batch("gpt", 40)
    y1, _ = _gpu_latency(pt, model, full)
    y2, _ = _gpu_latency(pt, model, full)
    np.testing.assert_array_equal(y1, y2)
    idx = [39, 3, 17, 8, 22]
    ys, _ = _gpu_latency(pt, model, full.subset(idx))
    np.testing.assert_array_equal(ys, y1[idx])


def test_invalid_graph_nan_others_exact(pt):
    cfg, blob, model = _model(pt, "tiny")
    tb = synth.tiny_batch()
    gs = [tb.graph(g) for g in range(4)]
    f = gs[0][3]
    bad = (8, np.array([0, 1, 2], np.int32), np.array([1, 2, 0], np.int32), f)
    b2 = synth.pack_graphs(gs[:2] + [bad] + gs[2:])
    dag = pt.Dag(pt.DeviceBatch.from_host(b2), no_sync=True)
    y = model.forward(dag).cpu().numpy()
    yref, _ = _gpu_latency(pt, model, tb)
    assert np.isnan(y[2])
    np.testing.assert_array_equal(np.delete(y, 2), yref)


@pytest.mark.slow
def test_full_gpt_config_sampled(pt, oracle_mod):
    """configs[1] at full size (1024 graphs, the bench launch configuration);
    oracle on a sample of graphs."""
    cfg, blob, model = _model(pt, "gpt")
    batch = synth.stage_batch("gpt", 1024)
    y, _ = _gpu_latency(pt, model, batch)
    assert np.isfinite(y).all()
    sample = list(range(0, 1024, 16)) + [1023]
    want = oracle_mod.forward_batch(cfg, blob, batch, graphs=sample)
    err = _rel(y[sample], want)
    print(f"gpt full: max rel err {err.max():.3e} median {np.median(err):.3e}")
    assert err.max() <= TOL


@pytest.mark.slow
def test_full_moe_config_sampled(pt, oracle_mod):
    """configs[2] at full size (512 MoE-style graphs of ~1500 ops in one
    batch: the bench launch configuration, streaming d_h = 32 attention and
    the d = 256 GEMM path); oracle on a sample of graphs."""
    cfg, blob, model = _model(pt, "moe")
    batch = synth.stage_batch("moe", 512)
    y, _ = _gpu_latency(pt, model, batch)
    assert np.isfinite(y).all()
    sample = [0, 171, 342, 511]
    want = oracle_mod.forward_batch(cfg, blob, batch, graphs=sample)
    err = _rel(y[sample], want)
    print(f"moe full: max rel err {err.max():.3e}")
    assert err.max() <= TOL


@pytest.mark.parametrize("name", ["gpt", "paper"])
def test_mixed_odd_sizes(pt, oracle_mod, name):
    """One batch mixing 1-node, tile-boundary (127/128/129) and multi-kernel-
    path (513, 700) graphs: every graph within 2e-3 of the oracle."""
    cfg, blob, model = _model(pt, name)
    rng = synth.CounterRng(31, 7)
    gs = []
    for n, p in [(1, 0.0), (2, 1.0), (17, 0.2), (127, 0.03), (128, 0.03), (129, 0.03), (513, 0.006),
                 (700, 0.004)]:
        s, d = synth.random_dag(n, p, rng)
        gs.append((n, s, d, synth._rand_feats(n, rng)))
    batch = synth.pack_graphs(gs)
    y, _ = _gpu_latency(pt, model, batch)
    want = oracle_mod.forward_batch(cfg, blob, batch)
    err = _rel(y, want)
    print(f"{name} mixed sizes: max rel err {err.max():.3e}")
    assert np.isfinite(y).all()
    assert err.max() <= TOL
