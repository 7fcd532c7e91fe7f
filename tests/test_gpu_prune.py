"""GPU parity of graph pruning (predtop_prune_graphs; SIV-B4, P:167-170;
reading R21) against the oracle: per graph the kept-node count, the edge list
(unique, sorted) and the node records are bit-exact; the pruned batch feeds
predtop_build_dag directly and scores exactly like the original stage graphs
(pruning inverts the splice of reshape / convert nodes)."""
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


def _raw_batch(seed=3):
    rng = synth.CounterRng(seed, 9)
    gs, orig = [], []
    b = synth.stage_batch("gpt", 6, first_graph=20)
    for g in range(b.num_graphs):
        n, s, d, f = b.graph(g)
        raw = synth.insert_pruned_ops(n, s, d, f, rng, frac=0.3)
        if g % 2:
            perm = rng.permutation(raw[0])
            raw = (raw[0],) + synth.relabel(raw[0], raw[1], raw[2], raw[3], perm)
        gs.append(raw)
        orig.append((n, s, d, f))
    n, s, d, f = synth.stage_batch("moe", 1).graph(0)  # a large graph (multi-kernel build path)
    gs.append(synth.insert_pruned_ops(n, s, d, f, rng, frac=0.2))
    orig.append((n, s, d, f))
    for n, p in [(1, 0.0), (40, 0.1), (130, 0.03)]:  # random DAGs, random removed subsets
        s, d = synth.random_dag(n, p, rng)
        f = synth._rand_feats(n, rng, kinds=[synth.KIND_OPERATOR] * n)
        for v in range(n):
            if rng.uniform() < 0.3:
                f[v]["op"] = synth.RAW_OP_CONVERT
        gs.append((n, s, d, f))
        orig.append(None)
    return synth.pack_graphs(gs), orig


def test_parity_vs_oracle(pt, oracle_mod):
    raw, _ = _raw_batch()
    out = pt.prune_graphs(pt.DeviceBatch.from_host(raw))
    torch.cuda.synchronize()
    onp = out.node_ptr.cpu().numpy()
    oep = out.edge_ptr.cpu().numpy()
    src, dst = out.src.cpu().numpy(), out.dst.cpu().numpy()
    feats = out.feats.cpu().numpy().view(synth.FEAT_DTYPE)
    for g in range(raw.num_graphs):
        n, s, d, f = raw.graph(g)
        st, nk, ws, wd, wf = oracle_mod.prune(n, s, d, f)
        assert st == oracle_mod.OK
        assert onp[g + 1] - onp[g] == nk, g
        np.testing.assert_array_equal(src[oep[g]:oep[g + 1]], ws, err_msg=f"src g={g}")
        np.testing.assert_array_equal(dst[oep[g]:oep[g + 1]], wd, err_msg=f"dst g={g}")
        assert feats[onp[g]:onp[g + 1]].tobytes() == wf.tobytes()


def test_pruned_graphs_score_like_the_originals(pt):
    raw, orig = _raw_batch(5)
    keep = [g for g, o in enumerate(orig) if o is not None and g % 2 == 0]  # unrelabelled stages
    rawk = raw.subset(keep)
    pruned = pt.prune_graphs(pt.DeviceBatch.from_host(rawk))
    cfg = dict(synth.MODEL_CONFIGS["gpt"])
    model = pt.Model(cfg, synth.pack_weights(cfg, synth.model_weights(cfg)))
    dag_p = pt.Dag(pruned)
    assert dag_p.status == pt.OK
    y_p = model.forward(dag_p).cpu()
    y_o = model.forward(pt.Dag(pt.DeviceBatch.from_host(synth.pack_graphs([orig[g] for g in keep])))).cpu()
    assert torch.equal(y_p, y_o)  # same DAG up to duplicate edges: bit-identical latencies


def test_capacity_retry_and_errors(pt):
    raw, _ = _raw_batch(7)
    db = pt.DeviceBatch.from_host(raw)
    a = pt.prune_graphs(db, edge_capacity=1)  # WORKSPACE -> retried with the exact count
    b = pt.prune_graphs(db)
    assert torch.equal(a.src.cpu(), b.src.cpu()) and torch.equal(a.edge_ptr.cpu(), b.edge_ptr.cpu())
    f = synth._rand_feats(3, synth.CounterRng(1, 1))
    cyc = synth.pack_graphs([(3, np.array([0, 1], np.int32), np.array([1, 2], np.int32), f),
                             (3, np.array([0, 1, 2], np.int32), np.array([1, 2, 0], np.int32), f)])
    with pytest.raises(pt.PredtopError) as e:
        pt.prune_graphs(pt.DeviceBatch.from_host(cyc))
    assert e.value.status == pt.CYCLE
