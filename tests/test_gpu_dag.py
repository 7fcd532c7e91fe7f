"""GPU parity of the DAG preprocessing (predtop_build_dag / predtop_reachability
/ debug mask + tiles) against the CPU oracle: bit-exact depth (DAGPE),
closure R incl. padding bits (DAGRA, P:135 / P:145), mask M = R | R^T | I,
tile classes and |A|.  Error reporting (RANGE / SELF_LOOP / CYCLE precedence)
and relabelling / duplicate-edge edge cases."""
import numpy as np
import pytest
import torch

from paper_conf_ipps_acharyas25_b200 import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pt():
    from paper_conf_ipps_acharyas25_b200 import build, predtop
    build.build_library()
    assert torch.cuda.is_available()
    return predtop


def _oracle_graph(oracle_mod, n, s, d):
    dep = oracle_mod.depth(n, s, d)
    R = oracle_mod.reach(n, s, d)
    M = oracle_mod.mask(n, R)
    cls, pairs = oracle_mod.tiles(n, M)
    return dep, R, M, cls, pairs


def _check_batch(pt, oracle_mod, batch, relabel_seed=None):
    db = pt.DeviceBatch.from_host(batch)
    dag = pt.Dag(db)
    assert dag.status == pt.OK, dag.status
    depth = dag.depth.cpu().numpy()
    R = dag.reachability().cpu().numpy().view(np.uint64)
    M = dag.mask().cpu().numpy().view(np.uint64)
    sizes = batch.sizes
    T = (sizes + 127) // 128
    cls, pairs = dag.tiles(int((T * T).sum()))
    cls, pairs = cls.cpu().numpy(), pairs.cpu().numpy()
    woff, toff = 0, 0
    for g in range(batch.num_graphs):
        n, s, d, _ = batch.graph(g)
        dep, Ro, Mo, co, po = _oracle_graph(oracle_mod, n, s, d)
        n0 = batch.node_ptr[g]
        np.testing.assert_array_equal(depth[n0:n0 + n], dep, err_msg=f"depth g={g}")
        W = oracle_mod.row_words(n)
        np.testing.assert_array_equal(R[woff:woff + n * W], Ro.ravel(), err_msg=f"R g={g}")
        np.testing.assert_array_equal(M[woff:woff + n * W], Mo.ravel(), err_msg=f"M g={g}")
        np.testing.assert_array_equal(cls[toff:toff + len(co)], co, err_msg=f"tiles g={g}")
        assert pairs[g] == po
        woff += n * W
        toff += len(co)
    assert woff == len(R) or (woff == 0 and len(R) == 1)
    return dag


def test_tiny(pt, oracle_mod):
    _check_batch(pt, oracle_mod, synth.tiny_batch())


def test_gpt_batch(pt, oracle_mod):
    _check_batch(pt, oracle_mod, synth.stage_batch("gpt", 48))


def test_moe_batch(pt, oracle_mod):
    _check_batch(pt, oracle_mod, synth.stage_batch("moe", 4))


def test_16k_graph(pt, oracle_mod):
    _check_batch(pt, oracle_mod, synth.stage_batch("16k", 1))


def test_random_relabelled_and_edge_cases(pt, oracle_mod):
    rng = synth.CounterRng(42, 1)
    gs = []
    for n, p in [(1, 0.0), (2, 1.0), (63, 0.05), (64, 0.05), (65, 0.05), (127, 0.03), (128, 0.03),
                 (129, 0.03), (200, 0.0), (257, 0.02), (300, 0.3)]:
        s, d = synth.random_dag(n, p, rng)
        gs.append((n, s, d, synth._rand_feats(n, rng)))
    # duplicates + isolated nodes
    gs.append((6, np.array([0, 0, 1, 1, 3], np.int32), np.array([1, 1, 2, 2, 4], np.int32),
               synth._rand_feats(6, rng)))
    # a relabelled real stage graph
    n, s, d, f = synth.stage_batch("gpt", 1, first_graph=7).graph(0)
    s2, d2, f2 = synth.relabel(n, s, d, f, rng.permutation(n))
    gs.append((n, s2, d2, f2))
    _check_batch(pt, oracle_mod, synth.pack_graphs(gs))


def test_errors_reported(pt):
    f = synth._rand_feats(4, synth.CounterRng(1, 1))
    good = (4, np.array([0, 1], np.int32), np.array([1, 2], np.int32), f)
    cyc = (4, np.array([0, 1, 2], np.int32), np.array([1, 2, 0], np.int32), f)
    loop = (4, np.array([0, 1, 3, 2], np.int32), np.array([1, 1, 3, 0], np.int32), f)
    rng_ = (4, np.array([0, 7, 1], np.int32), np.array([1, 2, 1], np.int32), f)
    for gs, want, first in [([good, cyc, good], pt.CYCLE, 1), ([good, good, loop, cyc], pt.SELF_LOOP, 2),
                            ([rng_, cyc], pt.RANGE, 0), ([good, good], pt.OK, -1)]:
        dag = pt.Dag(pt.DeviceBatch.from_host(synth.pack_graphs(gs)))
        assert dag.status == want and dag.first_bad == first
        dep = dag.depth.cpu().numpy().reshape(-1, 4)
        for g, gr in enumerate(gs):
            if gr is good:
                np.testing.assert_array_equal(dep[g], [0, 1, 2, 0])  # other graphs unaffected
            else:
                assert (dep[g] == -1).all()


def test_no_sync_status_later(pt):
    f = synth._rand_feats(3, synth.CounterRng(2, 2))
    b = synth.pack_graphs([(3, np.array([0], np.int32), np.array([1], np.int32), f),
                           (3, np.array([0, 1, 2], np.int32), np.array([1, 2, 0], np.int32), f)])
    dag = pt.Dag(pt.DeviceBatch.from_host(b), no_sync=True)
    assert dag.status == pt.OK and dag.first_bad == -1
    st, bad = dag.dag_status()
    assert st == pt.CYCLE and bad == 1


def test_rebuild_deterministic(pt):
    b = synth.stage_batch("gpt", 16, first_graph=100)
    dag = pt.Dag(pt.DeviceBatch.from_host(b))
    R1 = dag.reachability().cpu()
    d1 = dag.depth.clone()
    assert dag.rebuild() == pt.OK
    assert torch.equal(R1, dag.reachability().cpu())
    assert torch.equal(d1, dag.depth)


@pytest.mark.parametrize("n", [6780, 9000])
def test_large_graph_column_slicing(pt, oracle_mod, n):
    """Graphs between the fused path and the 16k stress case on the deep-graph
    record path: n = 6780 gives W = 106 words in three-word shared-memory
    slices, the last slice one word wide (its row stride is still 3) and
    holding real columns 6720..6779."""
    rng = synth.CounterRng(n, 17)
    s, d = synth.random_dag(n, 1.6 / n, rng)
    b = synth.pack_graphs([(n, s, d, synth._rand_feats(n, rng))])
    dag = pt.Dag(pt.DeviceBatch.from_host(b))
    assert dag.status == pt.OK
    R = dag.reachability().cpu().numpy().view(np.uint64)
    np.testing.assert_array_equal(R, oracle_mod.reach(n, s, d).ravel())
    np.testing.assert_array_equal(dag.depth.cpu().numpy(), oracle_mod.depth(n, s, d))


@pytest.mark.parametrize("n, kind", [(520, "random"), (3000, "random"), (4100, "chain"), (7000, "chain"),
                                     (12000, "random")])
def test_large_path_modes(pt, oracle_mod, n, kind):
    """Multi-kernel build path across the column-slice modes (CSR staged in
    shared memory or not, 1-4 word columns per CTA, deep chains with one
    node per level): depth, R and the mask tiles bit-exact."""
    rng = synth.CounterRng(n, 23)
    if kind == "chain":
        s, d = synth.chain(n)
        perm = rng.permutation(n)
        s, d = perm[s].astype(np.int32), perm[d].astype(np.int32)
    else:
        s, d = synth.random_dag(n, 2.0 / n, rng)
    b = synth.pack_graphs([(n, s, d, synth._rand_feats(n, rng))])
    dag = pt.Dag(pt.DeviceBatch.from_host(b))
    assert dag.status == pt.OK
    R = dag.reachability().cpu().numpy().view(np.uint64)
    Ro = oracle_mod.reach(n, s, d)
    np.testing.assert_array_equal(R, Ro.ravel())
    np.testing.assert_array_equal(dag.depth.cpu().numpy(), oracle_mod.depth(n, s, d))
    T = (n + 127) // 128
    cls, pairs = dag.tiles(T * T)
    co, po = oracle_mod.tiles(n, oracle_mod.mask(n, Ro))
    np.testing.assert_array_equal(cls.cpu().numpy(), co)
    assert int(pairs.cpu()[0]) == po
