"""GPU parity of the inter-stage plan search (predtop_plan_search; SURVEY 8(f)
f1, reading R20) against the oracle's exhaustive enumeration: T* bit-exact
(dyadic latencies keep the fp64 sums exact), the returned plan valid (covers
the layers contiguously, uses exactly D devices, feasible stages) with its
Eqn 4 equal to T*, +inf when no plan exists, NaN for invalid problems."""
import math
import os

import numpy as np
import pytest
import torch

from paper_conf_ipps_acharyas25_b200 import synth

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module")
def pt():
    from paper_conf_ipps_acharyas25_b200 import build, predtop
    build.build_library()
    assert torch.cuda.is_available()
    return predtop


def _run(pt, tables, dev, D, Bs, table_of=None, pad=0):
    tables = np.ascontiguousarray(tables, np.float32)
    if tables.ndim == 3:
        tables = tables[None]
    L = tables.shape[1]
    packed = np.stack([pt.pack_stage_table(t) for t in tables])
    if pad:  # rows with a stride beyond L(L+1)/2 (all-gather layouts)
        packed = np.concatenate([packed, np.full(packed.shape[:2] + (pad,), -1.0, np.float32)], axis=2)
    ps = pt.PlanSearch(len(Bs), L, dev, D)
    t = torch.from_numpy(np.ascontiguousarray(packed)).cuda()
    B = torch.tensor(Bs, dtype=torch.int32, device="cuda")
    to = None if table_of is None else torch.tensor(table_of, dtype=torch.int32, device="cuda")
    ps.run(t, B, to)
    torch.cuda.synchronize()
    return ps.plans()


def _valid(oracle_mod, t, dev, D, B, T, stages):
    L = t.shape[0]
    assert stages[0][0] == 0 and stages[-1][1] == L - 1
    for (_, b0, _), (a1, _, _) in zip(stages, stages[1:]):
        assert a1 == b0 + 1
    assert sum(dev[c] for _, _, c in stages) == D
    lat = np.asarray([t[i, j, c] for i, j, c in stages], np.float32)
    assert np.isfinite(lat).all() and (lat >= 0).all()
    assert oracle_mod.plan_T([0, len(stages)], list(range(len(stages))), [B], lat)[0] == T


def _table(a, choices):
    L = len(a)
    t = np.full((L, L, len(choices)), np.inf, np.float32)
    for i in range(L):
        for j in range(i, L):
            for c, (_, scale, off) in enumerate(choices):
                t[i, j, c] = scale * sum(a[i:j + 1]) + off
    return t


def test_golden(pt, oracle_mod):
    for line in open(os.path.join(HERE, "golden", "plan_search.txt")):
        line = line.split("#")[0].strip()
        if not line:
            continue
        f = [x.strip() for x in line.split(";")]
        D, B = map(int, f[0].split())
        a = [float(x) for x in f[1].split()]
        ch = [tuple(float(y) for y in x.split(":")) for x in f[2].split()]
        dev = [int(c[0]) for c in ch]
        t = _table(a, ch)
        (T, st), = _run(pt, t, dev, D, [B])
        assert T == float(f[3])
        if math.isinf(T):
            assert st == []
        else:
            _valid(oracle_mod, t, dev, D, B, T, st)


def _dyadic(rng, L, K, p_inf):
    t = np.full((L, L, K), np.inf, np.float32)
    for i in range(L):
        for j in range(i, L):
            for c in range(K):
                if rng.uniform() >= p_inf:
                    t[i, j, c] = rng.randint(1, 4097) / 64.0
    return t


@pytest.mark.parametrize("seed", range(6))
def test_random_vs_exhaustive(pt, oracle_mod, seed):
    rng = synth.CounterRng(500 + seed, 1)
    L = rng.randint(2, 13)
    K = rng.randint(1, 5)
    dev = [rng.choice([1, 2, 4]) for _ in range(K)]
    tables = np.stack([_dyadic(rng, L, K, 0.15) for _ in range(3)])
    probs = [(tb, D, B) for tb in range(3) for D in (1, 2, 4) for B in (1, 2, 16, 64)]
    for D in (1, 2, 4):
        sub = [(tb, B) for tb, d, B in probs if d == D]
        got = _run(pt, tables, dev, D, [B for _, B in sub], [tb for tb, _ in sub], pad=seed % 3 * 5)
        for (tb, B), (T, st) in zip(sub, got):
            Tw, _ = oracle_mod.plan_search(tables[tb], dev, D, B)
            assert T == Tw, (seed, tb, D, B)
            if math.isinf(T):
                assert st == []
            else:
                _valid(oracle_mod, tables[tb], dev, D, B, T, st)


def test_paper_meshes_gpt24(pt, oracle_mod):
    """Table II/III choices (1 GPU; 2 GPUs DP or MP; 4 GPUs DP, DP+MP, MP) on
    Platform 2's 4 GPUs, 24 layers (Table IV GPT-3)."""
    rng = synth.CounterRng(9, 24)
    L, dev = 24, [1, 2, 2, 4, 4, 4]
    a = [rng.randint(64, 129) / 64.0 for _ in range(L)]
    t = np.full((L, L, 6), np.inf, np.float32)
    eff = [1.0, 0.5, 0.625, 0.25, 0.3125, 0.375]
    for i in range(L):
        for j in range(i, L):
            s = sum(a[i:j + 1])
            for c in range(6):
                v = s * eff[c] + (j - i + 1) / 32.0 * (c > 0)
                if dev[c] == 1 and j - i + 1 > 12:
                    v = np.inf  # does not fit one GPU
                t[i, j, c] = v
    Bs = [1, 2, 4, 8, 16, 32, 64]
    got = _run(pt, t, dev, 4, Bs, [0] * len(Bs))
    for B, (T, st) in zip(Bs, got):
        Tw, _ = oracle_mod.plan_search(t, dev, 4, B)
        assert T == Tw
        _valid(oracle_mod, t, dev, 4, B, T, st)


def test_invalid_problems(pt):
    t = np.ones((2, 3, 3, 1), np.float32)
    got = _run(pt, t, [1], 1, [4, 0, 4], [0, 0, 5])
    assert got[0][0] == 4.0 and got[0][1] == [(0, 2, 0)]  # one stage on the 1 device: B * t[0][2]
    assert math.isnan(got[1][0]) and got[1][1] == []
    assert math.isnan(got[2][0]) and got[2][1] == []
    with pytest.raises(pt.PredtopError):
        _run(pt, t, [0], 1, [4])


def test_stage_table_end_to_end(pt, oracle_mod):
    """The f1 flow on one GPU: every layer-range stage of a 6-layer GPT model
    scored by 2 mesh models straight into the stage table (<= 2e-3 against
    the oracle forward), then the plan search on that table == the oracle's
    exhaustive search over the same table, bit for bit."""
    from paper_conf_ipps_acharyas25_b200 import stage_table
    L = 6
    host = synth.layer_range_stages("gpt", L)
    cfgs = synth.mesh_model_configs("search", 2)
    blobs = [synth.pack_weights(c, synth.model_weights(c)) for c in cfgs]
    dev, Bs = [1, 2], [1, 4, 16]
    sts = stage_table.StageTableSearch(pt, cfgs, blobs, host, L, dev, 2, Bs)
    sts.step()
    torch.cuda.synchronize()
    table = sts.table[0].cpu().numpy()
    for c in range(2):
        want = oracle_mod.forward_batch(cfgs[c], blobs[c], host)
        err = np.abs(table[c] - want) / np.abs(want)
        assert (want > 0).all() and err.max() <= 2e-3, err.max()
    dense = np.full((L, L, 2), np.inf, np.float32)
    for i in range(L):
        for j in range(i, L):
            dense[i, j] = table[:, synth.tri_index(i, j, L)]
    for B, (T, st) in zip(Bs, sts.search.plans()):
        Tw, _ = oracle_mod.plan_search(dense, dev, 2, B)
        assert T == Tw
        _valid(oracle_mod, dense, dev, 2, B, T, st)


@pytest.mark.slow
def test_search_config_full_size_sampled(pt, oracle_mod):
    """The --config search workload at full size (300 layer-range stages of
    GPT-3's 24 layers x 6 mesh models): sampled table entries against the
    oracle forward, and the plan search on the GPU table == exhaustive
    enumeration on the same table."""
    from paper_conf_ipps_acharyas25_b200 import stage_table
    L = 24
    host = synth.layer_range_stages("gpt", L)
    cfgs = synth.mesh_model_configs("search", 6)
    blobs = [synth.pack_weights(c, synth.model_weights(c)) for c in cfgs]
    dev, Bs = [d for _, d in synth.MESH_CHOICES], [1, 16, 64]
    sts = stage_table.StageTableSearch(pt, cfgs, blobs, host, L, dev, 4, Bs)
    sts.step()
    torch.cuda.synchronize()
    table = sts.table[0].cpu().numpy()
    assert np.isfinite(table).all() and (table > 0).all()
    # stages of 1, 3, 6 and 4 layers (~190 to ~1100 ops) on four of the mesh models
    picks = [(0, [synth.tri_index(0, 0, L), synth.tri_index(0, 2, L)]), (2, [synth.tri_index(3, 8, L)]),
             (3, [synth.tri_index(10, 13, L)]), (5, [synth.tri_index(23, 23, L)])]
    for c, gs in picks:
        want = oracle_mod.forward_batch(cfgs[c], blobs[c], host, graphs=gs)
        err = np.abs(table[c, gs] - want) / np.abs(want)
        assert err.max() <= 2e-3, (c, err)
    dense = np.full((L, L, 6), np.inf, np.float32)
    for i in range(L):
        for j in range(i, L):
            dense[i, j] = table[:, synth.tri_index(i, j, L)]
    for B, (T, st) in zip(Bs, sts.search.plans()):
        Tw, _ = oracle_mod.plan_search(dense, dev, 4, B)
        assert T == Tw
        _valid(oracle_mod, dense, dev, 4, B, T, st)
