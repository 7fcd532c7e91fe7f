"""Multi-process (gloo, world size 2, CPU) tests of the sharding and gather
logic of the multi-GPU path (paper_conf_ipps_acharyas25_b200/shard.py).  The
per-shard plan latencies come from the oracle here (the kernels need a GPU);
what is tested is the partitioning, the padded all-gather of variable shards
and the global (T, plan id) argmin, which must equal the single-process result
bit for bit."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_acharyas25_b200 import shard, synth


def test_even_and_balanced_ranges():
    assert shard.even_ranges(10, 3) == [(0, 4), (4, 7), (7, 10)]
    assert shard.even_ranges(2, 4) == [(0, 1), (1, 2), (2, 2), (2, 2)]
    costs = [1, 1, 1, 1, 10, 1, 1, 1]
    r = shard.balanced_ranges(costs, 2)
    assert r[0][0] == 0 and r[-1][1] == 8 and r[0][1] == r[1][0]
    # contiguous, covering, and the heavy item does not leave one rank with ~everything
    for world in (1, 2, 3, 8):
        rr = shard.balanced_ranges(np.random.RandomState(world).rand(100), world)
        assert rr[0][0] == 0 and rr[-1][1] == 100
        assert all(a[1] == b[0] for a, b in zip(rr[:-1], rr[1:]))
        tot = [sum(np.random.RandomState(world).rand(100)[s:e]) for s, e in rr]
        assert max(tot) - min(tot) <= 2.0 + 1e-9  # within two items (each < 1)


def test_plan_costs():
    pp = np.array([0, 2, 3])
    n = np.array([10, 20, 30])
    c = shard.plan_costs(pp, n, d=4)
    f = lambda x: 24 * x * 16 + 16 * x * x
    assert c[0] == f(10) + f(20) and c[1] == f(30)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, result_q, t_stage, plan_ptr, plan_stage, B, ranges):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    s, e = ranges[rank]
    # this rank's plans: local CSR over its range
    pp = np.asarray(plan_ptr[s:e + 1]) - plan_ptr[s]
    ps = np.asarray(plan_stage[plan_ptr[s]:plan_ptr[e]])
    T_local = torch.from_numpy(oracle.plan_T(pp, ps, B[s:e], t_stage))
    counts = [b - a for a, b in ranges]
    T_all = shard.gather_plan_latency(T_local, counts)
    best = shard.argmin_by_T_then_id(T_all.numpy())
    result_q.put((rank, T_all.numpy().tobytes(), best))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("uneven", [False, True])
def test_gloo_world2_gather_matches_single_process(oracle_mod, uneven):
    ps = synth.random_plans(101 if uneven else 100, 40, seed=7, max_s=8)
    r = synth.CounterRng(3, 3)
    # dyadic latencies with repeats -> exact ties across shards
    t = np.asarray([r.randint(1, 9) / 8.0 for _ in range(40)], np.float32)
    T_ref = oracle_mod.plan_T(ps.plan_ptr, ps.plan_stage, ps.microbatches, t)
    best_ref = oracle_mod.argmin(T_ref)
    ranges = shard.even_ranges(ps.num_plans, 2)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(rk, 2, port, q, t, ps.plan_ptr, ps.plan_stage,
                                               ps.microbatches, ranges)) for rk in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(2)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    for rank, tb, best in res:
        assert tb == T_ref.tobytes()      # every rank holds the global T, bit-exact
        assert best == best_ref           # same global argmin (ties -> lower id)


def _table_worker(rank, world, port, result_q, dense_rows, ranges, dev, D, Bs):
    """One rank of the shared-stage-table flow (stage_table.py steps 3-4):
    write its own range of the [K][NT] table, sum-all-reduce, then run the
    plan search (oracle here) on the gathered table."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    K, NT = dense_rows.shape
    g0, g1 = ranges[rank]
    mine = torch.zeros((1, K, NT), dtype=torch.float32)
    mine[0, :, g0:g1] = torch.from_numpy(dense_rows[:, g0:g1])
    dist.all_reduce(mine)
    table = mine[0].numpy()
    L = int((np.sqrt(8 * NT + 1) - 1) / 2)
    dense = np.full((L, L, K), np.inf, np.float32)
    for i in range(L):
        for j in range(i, L):
            dense[i, j] = table[:, synth.tri_index(i, j, L)]
    res = [oracle.plan_search(dense, dev, D, B)[0] for B in Bs]
    result_q.put((rank, table.tobytes(), res))
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_world2_stage_table_allreduce(oracle_mod):
    from paper_conf_ipps_acharyas25_b200 import stage_table
    L, K = 7, 3
    NT = L * (L + 1) // 2
    r = synth.CounterRng(12, 12)
    rows = np.asarray([[r.randint(1, 200) / 32.0 for _ in range(NT)] for _ in range(K)], np.float32)
    sizes = [100 + 50 * i for i in range(NT)]
    ranges = shard.balanced_ranges(stage_table.stage_costs(sizes, 128), 2)
    want_table = stage_table.assemble_table_host([(a, b, rows[:, a:b]) for a, b in ranges], K, NT)
    np.testing.assert_array_equal(want_table, rows)
    dev, D, Bs = [1, 2, 4], 4, [1, 4, 16]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_table_worker, args=(rk, 2, port, q, rows, ranges, dev, D, Bs)) for rk in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(2)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    (_, t0, r0), (_, t1, r1) = res
    assert t0 == t1 == rows.tobytes()  # the sum of disjoint ranges is exact
    assert r0 == r1                    # replicated search: identical optima on every rank
