"""GPU parity of the DAG-Transformer forward (predtop_stage_forward) against the
CPU fp64 oracle, per graph relative error <= 2e-3 (BASELINE.json north star),
plus layer-wise taps (localisation), determinism and shard invariance
(per-graph outputs bit-identical whatever the batch composition)."""
import numpy as np
import pytest
import torch

from paper_conf_ipps_acharyas25_b200 import synth
from _parity import rel_err_stats

pytestmark = pytest.mark.gpu
TOL = 2e-3
# fp16 unit roundoff: every GEMM operand (x, q/k/v, P, attention output, FFN
# hidden) is rounded once to fp16 (R18), everything else is fp32
U16 = 2.0 ** -11


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
def test_latency_parity(pt, oracle_mod, parity_log, name, batch_fn):
    """Per-graph latency within 2e-3 of the oracle, also after removing the
    head's constant output bias c_o (R17), which would otherwise dilute the
    relative error of the computed part."""
    cfg, blob, model = _model(pt, name)
    batch = batch_fn()
    y, _ = _gpu_latency(pt, model, batch)
    want, cond = oracle_mod.forward_batch_cond(cfg, blob, batch)
    st = rel_err_stats(y, want, cond)
    parity_log(f"latency_parity[{name}]", **st)
    print(f"{name}: {st}")
    assert np.isfinite(y).all()
    assert st["max_rel"] <= TOL
    assert st["max_rel_nobias"] <= TOL


@pytest.mark.parametrize("name, batch_fn, tc", [
    ("paper", lambda: synth.stage_batch("gpt", 12, seed=11), "1"),
    ("gpt", lambda: synth.stage_batch("gpt", 24), "1"),
    ("gpt", lambda: synth.tiny_batch(), "1"),
    ("moe", lambda: synth.stage_batch("moe", 3, first_graph=20), "0"),
])
def test_latency_parity_attention_kernel_choice(pt, oracle_mod, parity_log, name, batch_fn, tc, monkeypatch):
    """The attention kernel that is NOT the default for the head dim:
    PREDTOP_ATTN_TC=1 runs the tcgen05/TMEM kernel (attention_tc.cu) at
    d_h = 16, =0 the mma.sync kernel (attention.cu) at d_h = 32."""
    monkeypatch.setenv("PREDTOP_ATTN_TC", tc)
    cfg, blob, model = _model(pt, name)
    batch = batch_fn()
    y, _ = _gpu_latency(pt, model, batch)
    want, cond = oracle_mod.forward_batch_cond(cfg, blob, batch)
    st = rel_err_stats(y, want, cond)
    parity_log(f"latency_parity_attn_tc={tc}[{name}]", **st)
    print(f"{name} (PREDTOP_ATTN_TC={tc}): {st}")
    assert np.isfinite(y).all()
    assert st["max_rel"] <= TOL and st["max_rel_nobias"] <= TOL


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


@pytest.mark.parametrize("tc", ["0", None])
@pytest.mark.parametrize("name, n", [("paper", 1700), ("moe", 800)])
def test_latency_parity_streaming_attention(pt, oracle_mod, name, n, tc, monkeypatch):
    """Graphs whose K/V do not fit shared memory (d_h = 16: N > 1536; d_h =
    32: N > 768) take the two-buffer TMA streaming path of the mma.sync
    attention kernel when it is forced (PREDTOP_ATTN_TC=0); by default the
    large graph goes to the tcgen05 kernel and the small one (90 nodes, d_h =
    16) to the mma.sync kernel: the per-graph split of one batch."""
    if tc is not None:
        monkeypatch.setenv("PREDTOP_ATTN_TC", tc)
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


@pytest.mark.parametrize("name, batch_fn", [
    ("gpt", lambda: synth.stage_batch("gpt", 3, first_graph=50)),
    ("moe", lambda: synth.stage_batch("moe", 2, first_graph=7)),
])
def test_layer_taps(pt, oracle_mod, parity_log, name, batch_fn):
    """Node embeddings layer by layer (d = 128 fused tail layer2.cu; d = 256 fused tail layer256.cu).
    x0 (fp32 embedding) within 1e-4.  Each layer CONDITIONALLY: the oracle
    layer applied to the GPU's own input of that layer, so the check sees one
    layer's rounding, not the accumulated drift.  Budget: the layer output is
    post-LN (unit scale); one layer rounds its operands to fp16 five times on
    the way (x, q/k/v, P, attention output, FFN hidden), each a relative
    perturbation <= u = 2^-11 that LN renormalises, so an element's error is
    O(u) with heavy-tailed maxima: RMS <= 2u, max <= 32u.  Cumulative taps
    (oracle end to end) within 64u max, since the per-layer errors add."""
    cfg, blob, model = _model(pt, name)
    b = batch_fn()
    dag = pt.Dag(pt.DeviceBatch.from_host(b))
    offs = np.concatenate([[0], np.cumsum(b.sizes)])
    taps = [oracle_mod.forward(cfg, blob, *b.graph(g), taps=True)[2] for g in range(b.num_graphs)]
    masks = []
    for g in range(b.num_graphs):
        n, s_, d_, _ = b.graph(g)
        masks.append(oracle_mod.mask(n, oracle_mod.reach(n, s_, d_)))
    xs = [model.node_embeddings(dag, layer).cpu().numpy().astype(np.float64)
          for layer in range(-1, cfg["num_layers"])]
    for layer in range(-1, cfg["num_layers"]):
        x = xs[layer + 1]
        cum = np.abs(x - np.concatenate([t[layer + 1] for t in taps])).max()
        if layer < 0:
            print(f"{name} x0: max abs err {cum:.3e}")
            parity_log(f"taps[{name}].x0", max_abs=cum)
            assert cum < 1e-4
            continue
        cond = []
        for g in range(b.num_graphs):
            n = int(b.sizes[g])
            xin = xs[layer][offs[g]:offs[g + 1]]
            want = oracle_mod.layer_rows(cfg, blob, layer, n, masks[g], xin)
            cond.append(x[offs[g]:offs[g + 1]] - want)
        cond = np.concatenate(cond)
        cmax, crms = np.abs(cond).max(), np.sqrt((cond ** 2).mean())
        print(f"{name} layer {layer}: conditional max {cmax / U16:.1f}u rms {crms / U16:.2f}u; "
              f"cumulative max {cum / U16:.1f}u")
        parity_log(f"taps[{name}].layer{layer}", cond_max_abs=cmax, cond_rms=crms, cum_max_abs=cum, u=U16)
        assert crms <= 2 * U16
        assert cmax <= 32 * U16
        assert cum <= 64 * U16


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
def test_full_gpt_config_sampled(pt, oracle_mod, parity_log):
    """configs[1] at full size (1024 graphs, the bench launch configuration);
    oracle on a sample of graphs."""
    cfg, blob, model = _model(pt, "gpt")
    batch = synth.stage_batch("gpt", 1024)
    y, _ = _gpu_latency(pt, model, batch)
    assert np.isfinite(y).all()
    sample = list(range(0, 1024, 16)) + [1023]
    want, cond = oracle_mod.forward_batch_cond(cfg, blob, batch, graphs=sample)
    st = rel_err_stats(y[sample], want, cond)
    parity_log("full_gpt_sampled", **st)
    print(f"gpt full: {st}")
    assert st["max_rel"] <= TOL and st["max_rel_nobias"] <= TOL


@pytest.mark.slow
def test_full_moe_config_sampled(pt, oracle_mod, parity_log):
    """configs[2] at full size (512 MoE-style graphs of ~1500 ops in one
    batch: the bench launch configuration, streaming d_h = 32 attention and
    the d = 256 GEMM path); oracle on a sample of graphs."""
    cfg, blob, model = _model(pt, "moe")
    batch = synth.stage_batch("moe", 512)
    y, _ = _gpu_latency(pt, model, batch)
    assert np.isfinite(y).all()
    sample = list(range(0, 512, 16)) + [511]  # 33 graphs
    want, cond = oracle_mod.forward_batch_cond(cfg, blob, batch, graphs=sample)
    st = rel_err_stats(y[sample], want, cond)
    parity_log("full_moe_sampled", **st)
    print(f"moe full: {st}")
    assert st["max_rel"] <= TOL and st["max_rel_nobias"] <= TOL


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


@pytest.mark.slow
def test_16k_forward_parity(pt, oracle_mod, parity_log):
    """configs[3]: the single 16 384-op stage DAG through all 4 layers against
    the oracle end to end (layers evaluated row block by row block on the host
    cores, oracle.forward_rows), plus the conditional last-layer check on a
    row sample (streaming attention over 256 key chunks per row)."""
    cfg, blob, model = _model(pt, "16k")
    b = synth.stage_batch("16k", 1)
    dag = pt.Dag(pt.DeviceBatch.from_host(b))
    y = model.forward(dag).cpu().numpy().astype(np.float64)
    n, s_, d_, f_ = b.graph(0)
    st_, want, taps16 = oracle_mod.forward_rows(cfg, blob, n, s_, d_, f_, taps=True)
    assert st_ == 0
    st = rel_err_stats(y, [want], [oracle_mod.head_condition(cfg, blob, n, taps16[-1])])
    parity_log("16k_forward", **st, y=float(y[0]), want=want)
    print(f"16k: y {y[0]:.6f} oracle {want:.6f} {st}")
    assert st["max_rel"] <= TOL and st["max_rel_nobias"] <= TOL
    L = cfg["num_layers"]
    xin = model.node_embeddings(dag, L - 2).cpu().numpy().astype(np.float64)
    xout = model.node_embeddings(dag, L - 1).cpu().numpy().astype(np.float64)
    rows = sorted(set(synth.CounterRng(16, 3).permutation(n)[:256].tolist()) | {0, n - 1})
    M = oracle_mod.mask(n, oracle_mod.reach(n, s_, d_))
    cond = xout[rows] - oracle_mod.layer_rows(cfg, blob, L - 1, n, M, xin, rows=rows)
    cmax, crms = np.abs(cond).max(), np.sqrt((cond ** 2).mean())
    parity_log("16k_last_layer_conditional", cond_max_abs=cmax, cond_rms=crms, rows=len(rows), u=U16)
    print(f"16k last layer: conditional max {cmax / U16:.1f}u rms {crms / U16:.2f}u")
    assert crms <= 2 * U16 and cmax <= 32 * U16


def test_sweep_chunk_4096(pt, oracle_mod, parity_log):
    """configs[4]'s launch shape: sweep.SweepShard scores 4096 stage graphs per
    build + forward (bench.py --chunk 4096).  64 sampled graphs of the chunk
    against the oracle; Eqn 4 over the GPU latencies bit-exact against the
    oracle's plan_T; the argmin against the oracle's."""
    from paper_conf_ipps_acharyas25_b200 import sweep
    cfg, blob, model = _model(pt, "gpt")
    pool = synth.stage_graphs_parallel("gpt", 1024)
    (p0, p1), pp, mb, s0, _ = sweep.shard_sweep(1200, 1, 0)
    sh = sweep.SweepShard(pt, model, pool, pp, mb, s0, chunk=4096)
    assert any(hi - lo == 4096 for lo, hi, _ in sh.chunks)
    T = sh.score()
    best = torch.empty(1, dtype=torch.int64, device="cuda")
    pt.predtop_plan_argmin(T, best)
    torch.cuda.synchronize()
    st_, bad = sh.status()
    assert st_ == pt.OK, (st_, bad)
    lat = sh.lat[:sh.num_stages].cpu().numpy()
    assert np.isfinite(lat).all()
    lo, hi, key = next(c for c in sh.chunks if c[1] - c[0] == 4096)
    idx = sorted(set(synth.CounterRng(4096, 1).permutation(4096)[:63].tolist()) | {4095})
    gs = [pool[(key[0] + i) % len(pool)] for i in idx]
    want, cond = oracle_mod.forward_batch_cond(cfg, blob, synth.pack_graphs(gs))
    got = lat[lo:hi][idx].astype(np.float64)
    st = rel_err_stats(got, want, cond)
    parity_log("sweep_chunk_4096", **st)
    print(f"sweep chunk: {st}")
    assert st["max_rel"] <= TOL and st["max_rel_nobias"] <= TOL
    Tw = oracle_mod.plan_T(pp, np.arange(sh.num_stages), mb, lat)
    assert T.cpu().numpy().tobytes() == Tw.tobytes()
    assert int(best.item()) == oracle_mod.argmin(Tw)


@pytest.mark.parametrize("name, tc", [("moe", "1"), ("gpt", "1")])
def test_attention_exact_row_fallback(pt, oracle_mod, parity_log, name, tc, monkeypatch):
    """tcgen05 attention (attention_tc.cu) with a peaked layer-0 attention:
    W_q and b_q of layer 0 scaled by 8 (exact in fp16), so on some rows an
    allowed score exceeds the diagonal (the kernel's fixed reference m) by
    16 or more in log2 units: P overflows fp16, the row sum is not finite and
    the row takes the exact CUDA-core path.
    Precondition checked on the oracle's own q, k; result within 2e-3."""
    monkeypatch.setenv("PREDTOP_ATTN_TC", tc)
    cfg = dict(synth.MODEL_CONFIGS[name])
    w = synth.model_weights(cfg)
    d, H = cfg["d_model"], cfg["num_heads"]
    dh = d // H
    w["L0.W_qkv"] = w["L0.W_qkv"].copy()
    w["L0.b_qkv"] = w["L0.b_qkv"].copy()
    w["L0.W_qkv"][:d] *= 8.0
    w["L0.b_qkv"][:d] *= 8.0
    blob = synth.pack_weights(cfg, w)
    model = pt.Model(cfg, blob)
    batch = synth.stage_batch(name, 2, first_graph=3)
    # precondition on graph 0, layer 0 (oracle fp64 q/k, log2 units)
    import ctypes
    n, s_, d_, f_ = batch.graph(0)
    x0 = oracle_mod.embed(cfg, blob, n, f_, oracle_mod.depth(n, s_, d_))
    qkv = np.zeros((n, 3 * d))
    oracle_mod.lib().orc_qkv_rows(ctypes.byref(oracle_mod.cfg(cfg)), oracle_mod._p(np.ascontiguousarray(blob, np.float32)),
                                  0, 0, n, oracle_mod._p(np.ascontiguousarray(x0)), oracle_mod._p(qkv))
    A = oracle_mod.bits_to_dense(oracle_mod.mask(n, oracle_mod.reach(n, s_, d_)), n).astype(bool)
    gap = 0.0
    for h in range(H):
        q = qkv[:, h * dh:(h + 1) * dh]
        k = qkv[:, d + h * dh:d + (h + 1) * dh]
        S = (q @ k.T) / np.sqrt(dh) / np.log(2.0)
        S = np.where(A, S, -np.inf)
        gap = max(gap, float((S.max(1) - np.diag(S)).max()))
    assert gap > 17.0, gap
    y, _ = _gpu_latency(pt, model, batch)
    want, cond = oracle_mod.forward_batch_cond(cfg, blob, batch)
    st = rel_err_stats(y, want, cond)
    parity_log(f"attention_exact_row_fallback[{name}]", gap_log2=gap, **st)
    print(f"{name} peaked attention (max gap {gap:.1f}): {st}")
    assert np.isfinite(y).all()
    assert st["max_rel"] <= TOL and st["max_rel_nobias"] <= TOL


@pytest.mark.parametrize("name, batch_fn", [
    ("moe", lambda: synth.stage_batch("moe", 2, first_graph=40)),
    ("gpt", lambda: synth.stage_batch("gpt", 6, first_graph=40)),
])
def test_latency_parity_unfused_gemm_path(pt, oracle_mod, parity_log, name, batch_fn, monkeypatch):
    """PREDTOP_UNFUSED=1: the three-GEMM layer path (O-proj + LN GEMM, FFN-1
    GEMM, FFN-2 + LN GEMM, gemm.cu) instead of the fused layer tail (layer2.cu
    at d = 128, layer256.cu at d = 256); the fallback for other widths."""
    monkeypatch.setenv("PREDTOP_UNFUSED", "1")
    cfg, blob, model = _model(pt, name)
    batch = batch_fn()
    y, _ = _gpu_latency(pt, model, batch)
    want, cond = oracle_mod.forward_batch_cond(cfg, blob, batch)
    st = rel_err_stats(y, want, cond)
    parity_log(f"latency_parity_unfused[{name}]", **st)
    print(f"{name} (unfused GEMM path): {st}")
    assert np.isfinite(y).all()
    assert st["max_rel"] <= TOL and st["max_rel_nobias"] <= TOL
