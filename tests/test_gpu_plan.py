"""GPU parity of the white-box pipeline model (predtop_plan_latency, Eqn 4,
P:200) and of the ranking: bit-exact T and identical argmin including exact
ties, given the same fp32 stage latencies (reading R13)."""
import itertools
import math

import numpy as np
import pytest
import torch

from paper_conf_ipps_acharyas25_b200 import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pt():
    from paper_conf_ipps_acharyas25_b200 import build, predtop
    build.build_library()
    return predtop


def test_random_plans_bit_exact(pt, oracle_mod):
    r = synth.CounterRng(9, 9)
    t = np.asarray([r.uniform() * 10 ** r.randint(-3, 3) for _ in range(500)], np.float32)
    ps = synth.random_plans(20000, 500, seed=3, max_s=64)
    plans = pt.Plans(ps.plan_ptr, ps.plan_stage, ps.microbatches)
    T, st, bad = plans.latency(torch.from_numpy(t).cuda())
    assert st == pt.OK and bad == -1
    want = oracle_mod.plan_T(ps.plan_ptr, ps.plan_stage, ps.microbatches, t)
    got = T.cpu().numpy()
    assert got.tobytes() == want.tobytes()
    assert int(plans.argmin()[0]) == oracle_mod.argmin(want)


def test_dyadic_permuted_ties(pt, oracle_mod):
    """Plans that are permutations of each other must tie exactly; the argmin
    then picks the lowest plan id."""
    t = np.asarray([0.5, 0.25, 0.75, 1.5, 0.125, 2.0], np.float32)
    ptr, st_ = [0], []
    Bs = []
    base = [[3, 1, 4], [0, 5, 2, 1], [2, 2, 2]]
    for b in base:
        for perm in itertools.permutations(b):
            st_ += list(perm)
            ptr.append(ptr[-1] + len(perm))
            Bs.append(4)
    plans = pt.Plans(ptr, st_, Bs)
    T, st, _ = plans.latency(torch.from_numpy(t).cuda())
    got = T.cpu().numpy()
    want = oracle_mod.plan_T(ptr, st_, Bs, t)
    assert got.tobytes() == want.tobytes()
    assert len(set(got[:6].tolist())) == 1
    best = int(plans.argmin()[0])
    assert best == oracle_mod.argmin(want) == int(np.argmin(got))


def test_golden_and_closed_forms(pt):
    rows = [(3, [2, 5, 3, 1], 21.0), (3, [1, 2, 1, 1], 9.0), (16, [4], 64.0), (1, [3, 1, 4, 1, 5], 14.0),
            (16, [2, 2, 2, 2], 38.0)]
    t = np.concatenate([np.asarray(r[1], np.float32) for r in rows])
    ptr = np.concatenate([[0], np.cumsum([len(r[1]) for r in rows])])
    plans = pt.Plans(ptr, np.arange(len(t)), [r[0] for r in rows])
    T, st, _ = plans.latency(torch.from_numpy(t).cuda())
    assert T.cpu().numpy().tolist() == [r[2] for r in rows]


def test_invalid_plans(pt):
    t = torch.tensor([1.0, 2.0], device="cuda")
    plans = pt.Plans([0, 2, 4, 6], [0, 1, 0, 7, 1, 1], [2, 1, 0])
    T, st, bad = plans.latency(t)
    assert st == pt.INVALID_ARG and bad == 1
    got = T.cpu().numpy()
    assert got[0] == 3.0 + 2.0 and math.isnan(got[1]) and math.isnan(got[2])
    T, st, bad = plans.latency(t, no_sync=True)
    assert st == pt.OK
    assert int(plans.argmin()[0]) == 0


def test_argmin_nan_and_empty(pt):
    plans = pt.Plans([0, 1], [0], [1])
    T = torch.tensor([float("nan"), 3.0, float("nan"), 3.0, 5.0], dtype=torch.float64, device="cuda")
    assert int(plans.argmin(T)[0]) == 1
    T = torch.tensor([float("nan")], dtype=torch.float64, device="cuda")
    assert int(plans.argmin(T)[0]) == -1
