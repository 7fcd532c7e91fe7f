"""Pins of the oracle's inter-stage plan search (reading R20):
the optimum of Eqn 4 over every slicing of L layers into contiguous
stages with a mesh choice per stage using exactly D devices (P:194, P:212-214,
P:222).  The oracle enumerates every plan; the pins are
  * hand-worked instances (tests/golden/plan_search.txt);
  * closed forms: one choice of D devices -> B * t[0][L-1]; B = 1 with an
    additive single-device table -> sum of the layer latencies;
  * a textbook routine: with an additive single-device table and D devices,
    T* = sum(a) + (B - 1) * LP(a, D), LP = the optimal linear partition of a
    into D contiguous parts (binary search over the answer, greedy check);
  * a different algorithm: Alpa's t_max enumeration with a dynamic program over
    (first layer, devices left) on random tables of dyadic latencies (sums
    exact in fp64, so equality is bit for bit);
  * the returned plan is valid and Eqn 4 of it (orc_plan_T) equals T*;
  * monotonicity: lowering a table entry never raises T*.
"""
import math
import os

import numpy as np
import pytest

from paper_conf_ipps_acharyas25_b200 import synth

HERE = os.path.dirname(os.path.abspath(__file__))


def _table(a, choices):
    L = len(a)
    t = np.full((L, L, len(choices)), np.inf, np.float32)
    for i in range(L):
        for j in range(i, L):
            s = sum(a[i:j + 1])
            for c, (_, scale, off) in enumerate(choices):
                t[i, j, c] = scale * s + off
    return t


def _golden():
    rows = []
    for line in open(os.path.join(HERE, "golden", "plan_search.txt")):
        line = line.split("#")[0].strip()
        if not line:
            continue
        f = [x.strip() for x in line.split(";")]
        D, B = map(int, f[0].split())
        a = [float(x) for x in f[1].split()]
        ch = [tuple(float(y) for y in x.split(":")) for x in f[2].split()]
        T = float(f[3])
        plan = []
        for p in f[4].split() if len(f) > 4 else []:
            rng, c = p.split(":")
            i, j = rng.split("-")
            plan.append((int(i), int(j), int(c)))
        rows.append((D, B, a, ch, T, plan))
    return rows


def _check_plan(oracle_mod, t, dev, D, B, T, stages):
    L = t.shape[0]
    assert stages[0][0] == 0 and stages[-1][1] == L - 1
    for (a0, b0, _), (a1, _, _) in zip(stages, stages[1:]):
        assert a1 == b0 + 1
    assert sum(dev[c] for _, _, c in stages) == D
    lat = np.asarray([t[i, j, c] for i, j, c in stages], np.float32)
    Tp = oracle_mod.plan_T([0, len(stages)], list(range(len(stages))), [B], lat)[0]
    assert Tp == T


def test_golden_hand_worked(oracle_mod):
    rows = _golden()
    assert len(rows) == 7
    for D, B, a, ch, T, plan in rows:
        t = _table(a, ch)
        dev = [int(c[0]) for c in ch]
        got, stages = oracle_mod.plan_search(t, dev, D, B)
        assert got == T, (a, ch, D, B)
        if math.isinf(T):
            assert stages == []
        else:
            assert stages == plan
            _check_plan(oracle_mod, t, dev, D, B, got, stages)


def _dyadic_table(rng, L, K, p_inf=0.1):
    t = np.full((L, L, K), np.inf, np.float32)
    for i in range(L):
        for j in range(i, L):
            for c in range(K):
                if rng.uniform() >= p_inf:
                    t[i, j, c] = rng.randint(1, 257) / 16.0  # dyadic: exact sums
    return t


def test_closed_forms(oracle_mod):
    rng = synth.CounterRng(3, 3)
    for L in (1, 3, 6):
        t = _dyadic_table(rng, L, 1, p_inf=0.0)
        for B in (1, 4, 16):
            T, st = oracle_mod.plan_search(t, [4], 4, B)
            assert T == B * float(t[0, L - 1, 0]) and st == [(0, L - 1, 0)]
        a = [rng.randint(1, 64) / 8.0 for _ in range(L)]
        for D in range(1, L + 1):
            T, st = oracle_mod.plan_search(_table(a, [(1, 1.0, 0.0)]), [1], D, 1)
            assert T == sum(a) and len(st) == D


def _linear_partition(a, D):
    """Smallest possible maximum part sum over splits of a into <= D contiguous
    parts (integer a): binary search over the answer with a greedy check."""
    lo, hi = max(a), sum(a)
    while lo < hi:
        mid = (lo + hi) // 2
        parts, cur = 1, 0
        for x in a:
            if cur + x > mid:
                parts, cur = parts + 1, x
            else:
                cur += x
        if parts <= D:
            hi = mid
        else:
            lo = mid + 1
    return lo


@pytest.mark.parametrize("seed", range(6))
def test_linear_partition(oracle_mod, seed):
    rng = synth.CounterRng(40 + seed, 1)
    L = rng.randint(3, 11)
    a = [rng.randint(1, 40) for _ in range(L)]
    t = _table(a, [(1, 1.0, 0.0)])
    for D in range(1, min(L, 5) + 1):
        for B in (2, 7, 64):
            T, st = oracle_mod.plan_search(t, [1], D, B)
            assert T == sum(a) + (B - 1) * _linear_partition(a, D), (a, D, B)
            _check_plan(oracle_mod, t, [1], D, B, T, st)


def _alpa_dp(t, dev, D, B):
    """Alpa-style search: for every candidate t_max, F(k, d) = least sum of stage
    latencies covering layers k..L-1 with exactly d devices and every stage
    <= t_max; T* = min over t_max of F(0, D) + (B - 1) * t_max."""
    L, _, K = t.shape
    feas = np.isfinite(t) & (t >= 0)
    best = math.inf
    for tm in sorted({float(x) for x in t[feas]}):
        F = [[math.inf] * (D + 1) for _ in range(L + 1)]
        F[L][0] = 0.0
        for k in range(L - 1, -1, -1):
            for d in range(1, D + 1):
                for j in range(k, L):
                    for c in range(K):
                        if feas[k, j, c] and t[k, j, c] <= tm and dev[c] <= d:
                            F[k][d] = min(F[k][d], float(t[k, j, c]) + F[j + 1][d - dev[c]])
        if F[0][D] < math.inf:
            best = min(best, F[0][D] + (B - 1) * tm)
    return best


@pytest.mark.parametrize("seed", range(8))
def test_random_tables_vs_alpa_dp(oracle_mod, seed):
    rng = synth.CounterRng(90 + seed, 2)
    L = rng.randint(2, 8)
    K = rng.randint(1, 4)
    dev = [rng.choice([1, 2, 4]) for _ in range(K)]
    t = _dyadic_table(rng, L, K)
    for D in (1, 2, 4):
        for B in (1, 3, 16):
            T, st = oracle_mod.plan_search(t, dev, D, B)
            assert T == _alpa_dp(t, dev, D, B)
            if st:
                _check_plan(oracle_mod, t, dev, D, B, T, st)
            else:
                assert math.isinf(T)


def test_monotone_in_table(oracle_mod):
    rng = synth.CounterRng(7, 7)
    t = _dyadic_table(rng, 6, 2, p_inf=0.0)
    dev = [1, 2]
    T0, _ = oracle_mod.plan_search(t, dev, 4, 8)
    for _ in range(20):
        i = rng.randint(0, 6)
        j = rng.randint(i, 6)
        c = rng.randint(0, 2)
        t2 = t.copy()
        t2[i, j, c] = t2[i, j, c] / 2
        assert oracle_mod.plan_search(t2, dev, 4, 8)[0] <= T0
