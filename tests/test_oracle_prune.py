"""Pins of the oracle's graph pruning (SIV-B4; reading R21):
operator nodes whose op is a pruned primitive (reshape, convert_element_type)
are removed and their inputs spliced to their consumers.

  * boolean matrix formula on every DAG with n <= 4 and every subset of
    removed nodes: E' = A_KK | A_KP (I | A_PP | A_PP^2 | ...) A_PK;
  * splice inverse: pruning a synthetic stage graph with reshape/convert nodes
    spliced in (single, chained, shared by several consumers, dangling) gives
    back the original graph (edges deduplicated and sorted, records equal),
    also under a random relabelling of the raw graph;
  * reachability among kept nodes is preserved (the pinned orc_reach);
  * non-operator nodes are never removed; a graph without pruned ops is only
    deduplicated and sorted; invalid raw graphs report their status.
"""
import itertools

import numpy as np
import pytest

from paper_conf_ipps_acharyas25_b200 import synth


def _feats(n, ops, kinds=None):
    f = np.zeros(n, synth.FEAT_DTYPE)
    f["op"] = ops
    f["kind"] = synth.KIND_OPERATOR if kinds is None else kinds
    f["dims"][:, 0] = np.arange(n) + 1
    return f


def _formula(n, A, removed):
    K = [v for v in range(n) if not removed[v]]
    P = [v for v in range(n) if removed[v]]
    Ai = A.astype(np.int64)
    star = np.eye(len(P), dtype=np.int64)
    App = Ai[np.ix_(P, P)]
    cur = np.eye(len(P), dtype=np.int64)
    for _ in range(len(P)):
        cur = (cur @ App > 0).astype(np.int64)
        star |= cur
    E = Ai[np.ix_(K, K)] > 0
    if P:
        E |= (Ai[np.ix_(K, P)] @ star @ Ai[np.ix_(P, K)]) > 0
    return E


@pytest.mark.parametrize("n", [2, 3, 4])
def test_exhaustive_vs_matrix_formula(oracle_mod, n):
    pairs = [(i, j) for i in range(n) for j in range(n) if i != j]
    checked = 0
    for mask in range(1 << len(pairs)):
        sel = [pairs[k] for k in range(len(pairs)) if mask >> k & 1]
        s = np.asarray([p[0] for p in sel], np.int32)
        d = np.asarray([p[1] for p in sel], np.int32)
        if oracle_mod.validate(n, s, d) != oracle_mod.OK:
            continue
        A = np.zeros((n, n), bool)
        A[s, d] = True
        for rm in itertools.product([0, 1], repeat=n):
            ops = np.where(np.asarray(rm) == 1, synth.RAW_OP_RESHAPE, 3)
            st, nk, s2, d2, f2 = oracle_mod.prune(n, s, d, _feats(n, ops))
            assert st == oracle_mod.OK and nk == n - sum(rm)
            E = np.zeros((nk, nk), bool)
            E[s2, d2] = True
            np.testing.assert_array_equal(E, _formula(n, A, rm))
            assert len(set(zip(s2.tolist(), d2.tolist()))) == len(s2)        # unique
            assert list(zip(s2, d2)) == sorted(zip(s2.tolist(), d2.tolist()))  # sorted
            checked += 1
    assert checked == {2: 3 * 4, 3: 25 * 8, 4: 543 * 16}[n]


def _dedup_sorted(s, d):
    e = sorted(set(zip(np.asarray(s).tolist(), np.asarray(d).tolist())))
    return np.asarray([a for a, _ in e], np.int32), np.asarray([b for _, b in e], np.int32)


@pytest.mark.parametrize("g", range(4))
def test_splice_inverse_on_stage_graphs(oracle_mod, g):
    b = synth.stage_batch("gpt", 1, first_graph=g)
    n, s, d, f = b.graph(0)
    rng = synth.CounterRng(60 + g, 1)
    n2, s2, d2, f2 = synth.insert_pruned_ops(n, s, d, f, rng, frac=0.35)
    assert n2 > n + 20
    st, nk, ps, pd, pf = oracle_mod.prune(n2, s2, d2, f2)
    assert st == oracle_mod.OK and nk == n
    ws, wd = _dedup_sorted(s, d)
    np.testing.assert_array_equal(ps, ws)
    np.testing.assert_array_equal(pd, wd)
    assert pf.tobytes() == np.asarray(f).tobytes()
    # relabelled raw graph: kept nodes renumbered in raw order
    perm = rng.permutation(n2)
    s3, d3, f3 = synth.relabel(n2, s2, d2, f2, perm)
    st, nk, ps, pd, pf = oracle_mod.prune(n2, s3, d3, f3)
    order = np.sort(perm[:n])          # raw ids of the kept nodes, ascending
    new = {int(r): i for i, r in enumerate(order)}
    ws, wd = _dedup_sorted([new[int(perm[a])] for a in s], [new[int(perm[b_])] for b_ in d])
    np.testing.assert_array_equal(ps, ws)
    np.testing.assert_array_equal(pd, wd)


def test_reachability_preserved(oracle_mod):
    rng = synth.CounterRng(8, 8)
    n = 90
    s, d = synth.random_dag(n, 0.05, rng)
    ops = np.asarray([synth.RAW_OP_CONVERT if rng.uniform() < 0.4 else 1 for _ in range(n)])
    f = _feats(n, ops)
    st, nk, ps, pd, pf = oracle_mod.prune(n, s, d, f)
    kept = np.nonzero(ops != synth.RAW_OP_CONVERT)[0]
    R = oracle_mod.bits_to_dense(oracle_mod.reach(n, s, d), n)[np.ix_(kept, kept)]
    R2 = oracle_mod.bits_to_dense(oracle_mod.reach(nk, ps, pd), nk)
    np.testing.assert_array_equal(R2, R)


def test_kinds_and_no_ops_and_errors(oracle_mod):
    # pruned op ids on input / literal / output nodes are kept
    f = _feats(4, [64, 64, 64, 64], kinds=[0, 1, 3, 2])
    st, nk, ps, pd, pf = oracle_mod.prune(4, [0, 1, 3], [3, 3, 2], f)
    assert nk == 3 and list(zip(ps, pd)) == [(0, 2), (1, 2)]
    # nothing to prune: deduplicated and sorted
    st, nk, ps, pd, pf = oracle_mod.prune(3, [1, 0, 1, 0], [2, 1, 2, 2], _feats(3, [1, 2, 3]))
    assert nk == 3 and list(zip(ps, pd)) == [(0, 1), (0, 2), (1, 2)]
    assert oracle_mod.prune(3, [0, 1, 2], [1, 2, 0], _feats(3, [1, 1, 1]))[0] == oracle_mod.CYCLE
    assert oracle_mod.prune(3, [0, 5], [1, 2], _feats(3, [1, 1, 1]))[0] == oracle_mod.RANGE
