"""Pins of the oracle's finite-k DAGRA.

Paper: Eqn 1's mask admits u iff u in N_k(v); "the constant k is also
defined, which is a hyperparameter, that specifies the neighborhood range for
attention calculation" (the paper itself uses k = inf).  Reading R19
(DESIGN.md): N_k(v) = nodes joined to v by a directed path of <= k edges, in
either direction; R_k[v] = {u != v : shortest directed path v ~> u has 1..k
edges}; M_k = R_k | R_k^T | I.

Pins (none re-types the oracle's BFS):
  * boolean matrix powers: R_k = A | A^2 | ... | A^k, exhaustively on every
    labelled DAG with n <= 4 and all 1024 upper-triangular DAGs on 5 nodes
    under random relabelling, for every k;
  * a library routine: scipy.sparse.csgraph.shortest_path (unweighted,
    directed) distances 1..k on random and synthetic stage DAGs;
  * closed forms: chain (|R_k| = sum_{j=1..k} (n-j)), diamond, star;
  * special cases: k = 1 is the deduplicated edge set, k >= longest path is
    the full closure R (P:145 k = inf), R_k grows monotonically in k;
  * the forward pass with k >= the longest path equals the k = inf pass bit
    for bit, and with finite k equals the composition of the pinned steps
    with the k-hop mask; a k-hop chain layer equals torch's
    TransformerEncoderLayer under the banded mask |i-j| <= k.
"""
import numpy as np
import pytest
import torch
from scipy.sparse import csr_matrix
from scipy.sparse.csgraph import shortest_path

from paper_conf_ipps_acharyas25_b200 import synth


def _adj(n, src, dst):
    A = np.zeros((n, n), dtype=bool)
    A[np.asarray(src, int), np.asarray(dst, int)] = True
    return A


def _powers_upto(A, k):
    """A | A^2 | ... | A^k by boolean matrix products."""
    Ai = A.astype(np.int64)
    P = Ai.copy()
    R = A.copy()
    for _ in range(k - 1):
        P = ((P @ Ai) > 0).astype(np.int64)
        R |= P > 0
    return R


def _dense(oracle_mod, B, n):
    return oracle_mod.bits_to_dense(B, n)


def _dags(n):
    pairs = [(i, j) for i in range(n) for j in range(n) if i != j]
    for mask in range(1 << len(pairs)):
        sel = [pairs[k] for k in range(len(pairs)) if mask >> k & 1]
        A = np.zeros((n, n), bool)
        for i, j in sel:
            A[i, j] = True
        P = np.eye(n, dtype=np.int64)
        for _ in range(n):
            P = (P @ A.astype(np.int64) > 0).astype(np.int64)
        if P.any():
            continue  # not nilpotent: has a cycle
        yield (np.asarray([p[0] for p in sel], np.int32), np.asarray([p[1] for p in sel], np.int32))


@pytest.mark.parametrize("n", [2, 3, 4])
def test_exhaustive_small_dags_vs_boolean_powers(oracle_mod, n):
    count = 0
    for src, dst in _dags(n):
        A = _adj(n, src, dst)
        for k in range(1, n + 1):
            Rk = _dense(oracle_mod, oracle_mod.reach(n, src, dst, hops=k), n)
            np.testing.assert_array_equal(Rk, _powers_upto(A, k), err_msg=f"k={k}")
        count += 1
    assert count == {2: 3, 3: 25, 4: 543}[n]


def test_upper_triangular_n5_relabelled(oracle_mod):
    pairs = [(i, j) for i in range(5) for j in range(i + 1, 5)]
    rng = synth.CounterRng(19, 5)
    for mask in range(1 << len(pairs)):
        sel = [pairs[k] for k in range(len(pairs)) if mask >> k & 1]
        perm = rng.permutation(5)
        src = np.asarray([perm[p[0]] for p in sel], np.int32)
        dst = np.asarray([perm[p[1]] for p in sel], np.int32)
        A = _adj(5, src, dst)
        for k in (1, 2, 3):
            Rk = _dense(oracle_mod, oracle_mod.reach(5, src, dst, hops=k), 5)
            np.testing.assert_array_equal(Rk, _powers_upto(A, k))


def _shortest(n, src, dst):
    A = csr_matrix((np.ones(len(src)), (np.asarray(src), np.asarray(dst))), shape=(n, n))
    return shortest_path(A, method="D", directed=True, unweighted=True)


@pytest.mark.parametrize("n, p, seed", [(70, 0.05, 1), (130, 0.02, 2), (200, 0.015, 3)])
def test_random_dags_vs_scipy_shortest_path(oracle_mod, n, p, seed):
    src, dst = synth.random_dag(n, p, synth.CounterRng(seed, 31))
    D = _shortest(n, src, dst)
    for k in (1, 2, 3, 5, 8):
        Rk = _dense(oracle_mod, oracle_mod.reach(n, src, dst, hops=k), n)
        want = (D >= 1) & (D <= k)
        np.testing.assert_array_equal(Rk, want, err_msg=f"k={k}")
        # padding bits past n stay zero (layout of include/predtop.h)
        B = oracle_mod.reach(n, src, dst, hops=k)
        assert int(np.unpackbits(B.view(np.uint8), axis=1, bitorder="little")[:, n:].sum()) == 0


def test_synthetic_stage_graph_vs_scipy(oracle_mod):
    b = synth.stage_batch("gpt", 2)
    for g in range(2):
        n, s, d, _ = b.graph(g)
        D = _shortest(n, s, d)
        for k in (1, 4, 16):
            Rk = _dense(oracle_mod, oracle_mod.reach(n, s, d, hops=k), n)
            np.testing.assert_array_equal(Rk, (D >= 1) & (D <= k))


def test_closed_forms(oracle_mod):
    for n in (1, 2, 9, 65, 130):
        s, d = synth.chain(n)
        for k in (1, 2, 3, 7, 64, 200):
            Rk = _dense(oracle_mod, oracle_mod.reach(n, s, d, hops=k), n)
            i, j = np.indices((n, n))
            np.testing.assert_array_equal(Rk, (j > i) & (j - i <= k))
            assert Rk.sum() == sum(n - t for t in range(1, min(k, n - 1) + 1))
    # diamond s -> {a, b} -> t: k = 1 gives the 4 edges, k >= 2 adds s ~> t
    s = np.asarray([0, 0, 1, 2], np.int32)
    d = np.asarray([1, 2, 3, 3], np.int32)
    assert _dense(oracle_mod, oracle_mod.reach(4, s, d, hops=1), 4).sum() == 4
    assert _dense(oracle_mod, oracle_mod.reach(4, s, d, hops=2), 4).sum() == 5
    # star 1 -> k: every k gives the k edges
    s = np.zeros(15, np.int32)
    d = np.arange(1, 16, dtype=np.int32)
    for k in (1, 2, 5):
        assert _dense(oracle_mod, oracle_mod.reach(16, s, d, hops=k), 16).sum() == 15


def test_special_cases_and_monotone(oracle_mod):
    n = 150
    src, dst = synth.random_dag(n, 0.03, synth.CounterRng(5, 5))
    # duplicate edges are idempotent
    src = np.concatenate([src, src[:10]]).astype(np.int32)
    dst = np.concatenate([dst, dst[:10]]).astype(np.int32)
    A = _adj(n, src, dst)
    R1 = _dense(oracle_mod, oracle_mod.reach(n, src, dst, hops=1), n)
    np.testing.assert_array_equal(R1, A)
    L = int(oracle_mod.depth(n, src, dst).max())  # longest path in edges
    Rinf = oracle_mod.reach(n, src, dst)
    np.testing.assert_array_equal(oracle_mod.reach(n, src, dst, hops=L), Rinf)
    np.testing.assert_array_equal(oracle_mod.reach(n, src, dst, hops=L + 5), Rinf)
    if L >= 2:
        assert not np.array_equal(oracle_mod.reach(n, src, dst, hops=L - 1), Rinf)
    prev = np.zeros((n, n), bool)
    for k in range(1, L + 1):
        cur = _dense(oracle_mod, oracle_mod.reach(n, src, dst, hops=k), n)
        assert (prev <= cur).all()
        prev = cur


def test_forward_large_k_equals_infinite(oracle_mod):
    cfg = dict(synth.MODEL_CONFIGS["paper"])
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    b = synth.stage_batch("gpt", 1)
    n, s, d, f = b.graph(0)
    L = int(oracle_mod.depth(n, s, d).max())
    st0, y0, t0 = oracle_mod.forward(cfg, blob, n, s, d, f, taps=True)
    st1, y1, t1 = oracle_mod.forward(cfg, blob, n, s, d, f, taps=True, hops=L)
    assert st0 == st1 == 0
    assert y0 == y1
    np.testing.assert_array_equal(t0, t1)
    _, y2, _ = oracle_mod.forward(cfg, blob, n, s, d, f, hops=2)
    assert y2 != y0  # a short range changes the prediction


def test_forward_k_composes_pinned_steps(oracle_mod):
    cfg = dict(synth.MODEL_CONFIGS["paper"])
    blob = synth.pack_weights(cfg, synth.model_weights(cfg))
    n = 60
    rng = synth.CounterRng(9, 9)
    s, d = synth.random_dag(n, 0.06, rng)
    f = synth._rand_feats(n, rng)
    k = 2
    M = oracle_mod.mask(n, oracle_mod.reach(n, s, d, hops=k))
    x = oracle_mod.embed(cfg, blob, n, f, oracle_mod.depth(n, s, d))
    for l in range(cfg["num_layers"]):
        x = oracle_mod.layer(cfg, blob, l, n, M, x)
    st, y, taps = oracle_mod.forward(cfg, blob, n, s, d, f, taps=True, hops=k)
    assert st == 0
    np.testing.assert_array_equal(taps[-1], x)
    assert y == oracle_mod.readout(cfg, blob, n, x)


def test_chain_k_hop_layer_vs_torch_banded(oracle_mod):
    """On a chain, M_k is the band |i - j| <= k: one layer of the oracle under
    the k-hop mask equals torch's TransformerEncoderLayer with that band."""
    cfg = dict(synth.MODEL_CONFIGS["tiny"])
    w = synth.model_weights(cfg)
    blob = synth.pack_weights(cfg, w)
    dm, H, dff = cfg["d_model"], cfg["num_heads"], cfg["d_ff"]
    n, k = 40, 3
    s, d = synth.chain(n)
    M = oracle_mod.mask(n, oracle_mod.reach(n, s, d, hops=k))
    i, j = np.indices((n, n))
    band = np.abs(i - j) <= k
    np.testing.assert_array_equal(_dense(oracle_mod, M, n), band)
    x = synth.CounterRng(4, 7).uniform_array(n * dm).reshape(n, dm) * 4 - 2
    got = oracle_mod.layer(cfg, blob, 0, n, M, x)
    enc = torch.nn.TransformerEncoderLayer(dm, H, dff, dropout=0.0, activation="relu",
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
        enc.train()
        want = enc(T(x)[None], src_mask=torch.from_numpy(~band))[0].numpy()
    np.testing.assert_allclose(got, want, rtol=1e-10, atol=1e-10)
