"""Pins of the oracle's graph steps (validation, depth, reachability, mask,
tile classes) against brute force, closed forms and invariants -- nothing here
re-types the oracle's own algorithm.

Paper: stage graphs are DAGs; DAGPE depth; DAGRA
reachability "a path from m to n or vice versa" with k = inf;
mask M of Eqn 1.
"""
import itertools

import numpy as np
import pytest

from paper_conf_ipps_acharyas25_b200 import synth


def _adj(n, src, dst):
    A = np.zeros((n, n), dtype=bool)
    A[np.asarray(src, int), np.asarray(dst, int)] = True
    return A


def _warshall(A):
    """Transitive closure by Warshall's algorithm (boolean)."""
    R = A.copy()
    n = len(A)
    for k in range(n):
        R = R | (R[:, k:k + 1] & R[k:k + 1, :])
    return R


def _power_closure(A):
    """Closure by boolean powers: R = A + A^2 + ... + A^n."""
    n = len(A)
    R = np.zeros_like(A)
    P = A.astype(np.int64)
    for _ in range(n):
        R |= P > 0
        P = (P @ A.astype(np.int64)) > 0
        P = P.astype(np.int64)
    return R


def _acyclic(A):
    """A DAG iff its adjacency matrix is nilpotent: A^n = 0."""
    n = len(A)
    P = np.eye(n, dtype=np.int64)
    for _ in range(n):
        P = (P @ A.astype(np.int64) > 0).astype(np.int64)
    return not P.any()


def _all_paths_depth(n, A):
    """depth(v) = max number of edges over ALL directed paths ending at v,
    found by enumerating every path (brute force, tiny n only)."""
    best = [0] * n

    def walk(v, length):
        best[v] = max(best[v], length)
        for w in np.nonzero(A[v])[0]:
            walk(int(w), length + 1)

    for s in range(n):
        walk(s, 0)
    return np.asarray(best, np.int32)


def _dense_bits(oracle_mod, B, n):
    return oracle_mod.bits_to_dense(B, n)


def _digraphs(n):
    pairs = [(i, j) for i in range(n) for j in range(n) if i != j]
    for mask in range(1 << len(pairs)):
        sel = [pairs[k] for k in range(len(pairs)) if mask >> k & 1]
        src = np.asarray([p[0] for p in sel], np.int32)
        dst = np.asarray([p[1] for p in sel], np.int32)
        yield src, dst


@pytest.mark.parametrize("n, n_dags", [(1, 1), (2, 3), (3, 25), (4, 543)])
def test_exhaustive_small_digraphs(oracle_mod, n, n_dags):
    """Every labelled digraph on n <= 4 nodes: acyclicity vs nilpotency, depth
    vs all-path enumeration, closure vs Warshall and boolean powers.  The DAG
    counts 1, 3, 25, 543 are the known numbers of labelled DAGs (OEIS A003024)."""
    count = 0
    for src, dst in _digraphs(n):
        A = _adj(n, src, dst)
        st = oracle_mod.validate(n, src, dst)
        if not _acyclic(A):
            assert st == oracle_mod.CYCLE
            continue
        assert st == oracle_mod.OK
        count += 1
        np.testing.assert_array_equal(oracle_mod.depth(n, src, dst), _all_paths_depth(n, A))
        R = _dense_bits(oracle_mod, oracle_mod.reach(n, src, dst), n)
        np.testing.assert_array_equal(R, _warshall(A))
        np.testing.assert_array_equal(R, _power_closure(A))
    assert count == n_dags


def test_all_upper_triangular_dags_n5_relabelled(oracle_mod):
    """All 2^10 DAGs on 5 nodes with edges i<j, each under a random relabelling."""
    pairs = [(i, j) for i in range(5) for j in range(i + 1, 5)]
    rng = synth.CounterRng(11, 5)
    for mask in range(1 << len(pairs)):
        sel = [pairs[k] for k in range(len(pairs)) if mask >> k & 1]
        perm = rng.permutation(5)
        src = np.asarray([perm[p[0]] for p in sel], np.int32)
        dst = np.asarray([perm[p[1]] for p in sel], np.int32)
        A = _adj(5, src, dst)
        assert oracle_mod.validate(5, src, dst) == oracle_mod.OK
        np.testing.assert_array_equal(oracle_mod.depth(5, src, dst), _all_paths_depth(5, A))
        R = _dense_bits(oracle_mod, oracle_mod.reach(5, src, dst), 5)
        np.testing.assert_array_equal(R, _warshall(A))


def test_closed_forms(oracle_mod):
    # chain_n: depth i, |R| = n(n-1)/2, M all-ones
    for n in (1, 2, 8, 64, 65, 128, 129, 300):
        s, d = synth.chain(n)
        np.testing.assert_array_equal(oracle_mod.depth(n, s, d), np.arange(n))
        R = oracle_mod.reach(n, s, d)
        assert int(sum(bin(int(x)).count("1") for x in R.ravel())) == n * (n - 1) // 2
        M = _dense_bits(oracle_mod, oracle_mod.mask(n, R), n)
        assert M.all()
    # star_k: centre depth 0, leaves 1, |R| = k
    s, d = synth.star(17)
    np.testing.assert_array_equal(oracle_mod.depth(17, s, d), [0] + [1] * 16)
    R = _dense_bits(oracle_mod, oracle_mod.reach(17, s, d), 17)
    assert R.sum() == 16 and R[0, 1:].all()
    # diamond s -> {a, b} -> t: depths 0,1,1,2; |R| = 5
    s = np.asarray([0, 0, 1, 2], np.int32)
    d = np.asarray([1, 2, 3, 3], np.int32)
    np.testing.assert_array_equal(oracle_mod.depth(4, s, d), [0, 1, 1, 2])
    R = _dense_bits(oracle_mod, oracle_mod.reach(4, s, d), 4)
    assert R.sum() == 5 and not R[1, 2] and not R[2, 1]
    M = _dense_bits(oracle_mod, oracle_mod.mask(4, oracle_mod.reach(4, s, d)), 4)
    assert not M[1, 2] and M.sum() == 4 + 2 * 5
    # antichain: M = I
    M = _dense_bits(oracle_mod, oracle_mod.mask(5, oracle_mod.reach(5, [], [])), 5)
    np.testing.assert_array_equal(M, np.eye(5, dtype=bool))


def test_errors_and_precedence(oracle_mod):
    assert oracle_mod.validate(3, [0, 5], [1, 2]) == oracle_mod.RANGE
    assert oracle_mod.validate(3, [0, -1], [1, 2]) == oracle_mod.RANGE
    assert oracle_mod.validate(3, [0, 1], [1, 1]) == oracle_mod.SELF_LOOP
    assert oracle_mod.validate(3, [0, 1, 2], [1, 2, 0]) == oracle_mod.CYCLE
    # precedence: range beats self-loop beats cycle
    assert oracle_mod.validate(3, [0, 1, 2, 1, 0], [1, 2, 0, 1, 9]) == oracle_mod.RANGE
    assert oracle_mod.validate(3, [0, 1, 2, 1], [1, 2, 0, 1]) == oracle_mod.SELF_LOOP
    # duplicates and isolated nodes are fine
    assert oracle_mod.validate(4, [0, 0], [1, 1]) == oracle_mod.OK


@pytest.mark.parametrize("n, p", [(40, 0.08), (130, 0.02), (257, 0.01)])
def test_partial_order_invariants(oracle_mod, n, p):
    rng = synth.CounterRng(3, n)
    s, d = synth.random_dag(n, p, rng)
    A = _adj(n, s, d)
    Rb = oracle_mod.reach(n, s, d)
    R = _dense_bits(oracle_mod, Rb, n)
    np.testing.assert_array_equal(R, _warshall(A))
    assert not R.diagonal().any()                      # irreflexive
    assert not (R & R.T).any()                         # antisymmetric
    RR = (R.astype(np.int64) @ R.astype(np.int64)) > 0
    assert not (RR & ~R).any()                         # transitive
    # padding bits beyond n are zero
    full = np.unpackbits(Rb.view(np.uint8).reshape(n, -1), axis=1, bitorder="little")
    assert not full[:, n:].any()
    # edge reversal gives R^T, and the mask is unchanged
    Rr = _dense_bits(oracle_mod, oracle_mod.reach(n, d, s), n)
    np.testing.assert_array_equal(Rr, R.T)
    np.testing.assert_array_equal(oracle_mod.mask(n, Rb), oracle_mod.mask(n, oracle_mod.reach(n, d, s)))
    # relabelling: R permutes, depth permutes, popcounts invariant
    perm = rng.permutation(n)
    s2, d2 = perm[s].astype(np.int32), perm[d].astype(np.int32)
    R2 = _dense_bits(oracle_mod, oracle_mod.reach(n, s2, d2), n)
    inv = np.argsort(perm)
    np.testing.assert_array_equal(R2[np.ix_(perm, perm)], R)
    np.testing.assert_array_equal(oracle_mod.depth(n, s2, d2)[perm], oracle_mod.depth(n, s, d))
    assert inv is not None


def test_depth_equals_longest_path_dp_on_synthetic_stage(oracle_mod):
    """Depth against an independent longest-path DP over a topological order
    (numpy, Kahn order) on a real synthetic stage graph."""
    b = synth.stage_batch("gpt", 2)
    for g in range(2):
        n, s, d, f = b.graph(g)
        indeg = np.bincount(d, minlength=n)
        order, frontier = [], [v for v in range(n) if indeg[v] == 0]
        succ = [[] for _ in range(n)]
        for a, c in zip(s, d):
            succ[a].append(c)
        indeg = indeg.copy()
        while frontier:
            v = frontier.pop()
            order.append(v)
            for w in succ[v]:
                indeg[w] -= 1
                if indeg[w] == 0:
                    frontier.append(w)
        lp = np.zeros(n, np.int64)
        for v in order:
            for w in succ[v]:
                lp[w] = max(lp[w], lp[v] + 1)
        np.testing.assert_array_equal(oracle_mod.depth(n, s, d), lp)


def test_tiles_brute_force(oracle_mod):
    for n, p in [(5, 0.3), (128, 0.02), (129, 0.02), (300, 0.004)]:
        s, d = synth.random_dag(n, p, synth.CounterRng(9, n))
        M = oracle_mod.mask(n, oracle_mod.reach(n, s, d))
        cls, pairs = oracle_mod.tiles(n, M)
        D = _dense_bits(oracle_mod, M, n)
        assert pairs == int(D.sum())
        T = (n + 127) // 128
        for qt, kt in itertools.product(range(T), range(T)):
            blk = D[qt * 128:(qt + 1) * 128, kt * 128:(kt + 1) * 128]
            want = 0 if not blk.any() else (2 if blk.all() else 1)
            assert cls[qt * T + kt] == want
        R = _dense_bits(oracle_mod, oracle_mod.reach(n, s, d), n)
        assert pairs == n + 2 * int(R.sum())  # |A| = N + 2|R|
