"""Pins of the oracle's white-box pipeline model, Eqn 4 (SV):
  * brute force: the flow-shop recurrence implied by P:196 (microbatch b of
    stage i waits for microbatch b of stage i-1 and microbatch b-1 of stage i)
    gives the makespan C(S, B) = Eqn 4 exactly on integer inputs;
  * closed forms S = 1 -> B t, B = 1 -> sum t, all equal -> (S + B - 1) t;
  * the hand-worked Fig. 6-shaped golden rows (tests/golden/fig6_pipeline.txt);
  * R13: T depends only on the multiset of stage latencies (bit-identical
    under every permutation), ranking ties broken by the lower plan id.
"""
import itertools
import math
import os

import numpy as np
import pytest

from paper_conf_ipps_acharyas25_b200 import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "fig6_pipeline.txt")


def _flow_shop(t, B):
    S = len(t)
    C = [[0.0] * (B + 1) for _ in range(S + 1)]
    for i in range(1, S + 1):
        for b in range(1, B + 1):
            C[i][b] = max(C[i - 1][b], C[i][b - 1]) + t[i - 1]
    return C[S][B]


def _one(oracle_mod, t, B):
    return oracle_mod.plan_T([0, len(t)], np.arange(len(t)), [B], np.asarray(t, np.float32))[0]


def test_flow_shop_equivalence(oracle_mod):
    rng = synth.CounterRng(20000, 1)
    ptr, st, Bs, ts, want = [0], [], [], [], []
    for case in range(20000):
        S = rng.randint(1, 9)
        B = rng.randint(1, 20)
        t = [float(rng.randint(0, 1000)) for _ in range(S)]
        base = len(ts)
        ts += t
        st += list(range(base, base + S))
        ptr.append(ptr[-1] + S)
        Bs.append(B)
        want.append(_flow_shop(t, B))
    T = oracle_mod.plan_T(ptr, st, Bs, np.asarray(ts, np.float32))
    np.testing.assert_array_equal(T, np.asarray(want))


def test_closed_forms(oracle_mod):
    assert _one(oracle_mod, [3.5], 7) == 7 * 3.5                         # S = 1
    assert _one(oracle_mod, [1.0, 2.0, 4.0, 8.0], 1) == 15.0             # B = 1
    for S in range(1, 9):
        for B in (1, 2, 5, 64):
            assert _one(oracle_mod, [0.375] * S, B) == (S + B - 1) * 0.375  # GPipe bubble


def test_golden_fig6(oracle_mod):
    rows = [l for l in open(GOLDEN) if l.strip() and not l.startswith("#")]
    assert len(rows) >= 5
    for row in rows:
        B, t, T = row.split(";")
        t = [float(x) for x in t.split()]
        assert _one(oracle_mod, t, int(B)) == float(T)
        assert _flow_shop(t, int(B)) == float(T)


def test_permutation_ties_bit_exact(oracle_mod):
    rng = synth.CounterRng(5, 5)
    for _ in range(50):
        S = rng.randint(2, 7)
        t = [np.float32(rng.uniform() * 10 ** rng.randint(-3, 4)) for _ in range(S)]
        B = rng.randint(1, 65)
        vals = {np.float64(_one(oracle_mod, [t[i] for i in perm], B)).tobytes()
                for perm in itertools.permutations(range(S))}
        assert len(vals) == 1


def test_canonical_sum_close_to_exact(oracle_mod):
    """The sorted fp64 sum of fp32 values is within a few ulps of the exactly
    rounded sum (math.fsum)."""
    rng = synth.CounterRng(6, 6)
    for _ in range(2000):
        S = rng.randint(1, 65)
        t = np.asarray([rng.uniform() * 10 ** rng.randint(-6, 6) for _ in range(S)], np.float32)
        T = _one(oracle_mod, t, 1)
        exact = math.fsum(float(x) for x in t)
        assert abs(T - exact) <= 4 * np.spacing(exact)


def test_invalid_plans_nan(oracle_mod):
    t = np.asarray([1.0, 2.0], np.float32)
    T = oracle_mod.plan_T([0, 0, 2, 4, 6, 71], [0, 1, 0, 5, 1, -1] + [0] * 65,
                          [1, 0, 1, 1, 1], t)
    assert math.isnan(T[0])   # S = 0
    assert math.isnan(T[1])   # B = 0
    assert math.isnan(T[2])   # stage index 5 out of range
    assert math.isnan(T[3])   # stage index -1
    assert math.isnan(T[4])   # S = 65 > 64


def test_argmin_ties_and_nan(oracle_mod):
    assert oracle_mod.argmin([3.0, 1.0, 1.0, 2.0]) == 1
    assert oracle_mod.argmin([np.nan, 5.0, np.nan, 5.0]) == 1
    assert oracle_mod.argmin([np.nan, np.nan]) == -1
    assert oracle_mod.argmin([]) == -1
