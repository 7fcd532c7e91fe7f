"""Plan sweep (BASELINE.json configs[4]; SURVEY §8a a9-a10, §8e owned mode).

A sweep scores many candidate pipeline plans.  In owned mode plan p owns its
stage graphs (global stage ids [first_p, first_p + S_p)), so the work is: score
every stage graph with the DAG Transformer (predtop_build_dag +
predtop_stage_forward), then evaluate Eqn 4 for every plan
(predtop_plan_latency), then take the argmin by (T, plan id)
(predtop_plan_argmin).  A sweep of 100k plans owns ~500k stage graphs, more than
one launch should hold, so the graphs go through the library in chunks of
`chunk` graphs; each chunk is a full build + forward writing its slice of the
stage-latency vector.

Synthetic stage content: generating 500k distinct graphs on the host takes
longer than scoring them, so global stage id s takes the content of pool graph
(s mod U) of a pool of U distinct GPT-style stage graphs (synth.stage_graph,
ids 0..U-1).  Every stage is still built and scored on the device; nothing is
cached between chunks.  Host logic and argument marshalling only -- the
arithmetic runs in libpredtop.
"""
from __future__ import annotations

from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

from . import synth


class SweepShard:
    """One rank's share of an owned-mode sweep: its plans (a contiguous range
    of global plan ids) and their stage graphs, scored in chunks.

    plan_ptr/microbatches: this rank's plans, CSR over LOCAL stage ids
    0..S_local-1; stage_global0: global id of local stage 0 (contents come
    from pool[(stage_global0 + i) % len(pool)])."""

    def __init__(self, pt, model, pool: Sequence[Tuple], plan_ptr: np.ndarray,
                 microbatches: np.ndarray, stage_global0: int, chunk: int = 4096,
                 device="cuda"):
        import torch
        self.pt, self.model = pt, model
        self.num_stages = int(plan_ptr[-1])
        self.chunk = chunk
        U = len(pool)
        self.batches: Dict[Tuple[int, int], object] = {}
        self.dags: Dict[Tuple[int, int], object] = {}
        self.chunks: List[Tuple[int, int, Tuple[int, int]]] = []  # (lo, hi, key)
        for lo in range(0, self.num_stages, chunk):
            hi = min(self.num_stages, lo + chunk)
            key = ((stage_global0 + lo) % U, hi - lo)
            if key not in self.batches:
                ids = [(key[0] + i) % U for i in range(key[1])]
                host = synth.pack_graphs([pool[i] for i in ids])
                db = pt.DeviceBatch.from_host(host, device=device)
                self.batches[key] = db
                self.dags[key] = pt.Dag(db, no_sync=True)
            self.chunks.append((lo, hi, key))
        # one forward workspace sized for the largest chunk
        big = max(self.dags.values(), key=lambda d: d.batch.total_nodes)
        self.ws = model.forward_workspace(big)
        self.lat = torch.empty(max(self.num_stages, 1), dtype=torch.float32, device=device)
        self.plans = pt.Plans(plan_ptr, np.arange(self.num_stages, dtype=np.int32), microbatches,
                              device=device)

    @property
    def num_plans(self) -> int:
        return self.plans.num_plans

    def score(self):
        """Build + score every chunk, then Eqn 4 over this rank's plans.
        Returns the device tensor T of this rank's plans (fp64)."""
        for lo, hi, key in self.chunks:
            dag = self.dags[key]
            dag.rebuild()                                   # predtop_build_dag (NO_SYNC)
            self.model.forward(dag, self.ws, self.lat[lo:hi])  # predtop_stage_forward
        T, _, _ = self.plans.latency(self.lat, no_sync=True)  # predtop_plan_latency
        return T

    def status(self):
        """First DAG-build error over the chunks (OK if none); syncs."""
        for _, _, key in self.chunks:
            st, bad = self.dags[key].dag_status()
            if st != self.pt.OK:
                return st, bad
        return self.pt.OK, -1


def shard_sweep(num_plans: int, world: int, rank: int, seed: int = 4):
    """Rank `rank`'s plans of a sweep of `num_plans`, balanced by estimated cost
    (shard.balanced_ranges over the per-plan stage count; the stage graphs are
    all GPT-sized).  Returns (plan range (p0, p1), local plan_ptr, microbatches,
    global id of the first local stage, counts per rank)."""
    from . import shard
    ps, first = synth.sweep_plans(num_plans, seed=seed)
    S = np.diff(ps.plan_ptr).astype(np.float64)
    ranges = shard.balanced_ranges(S, world)
    p0, p1 = ranges[rank]
    pp = ps.plan_ptr[p0:p1 + 1] - ps.plan_ptr[p0]
    return (p0, p1), pp.astype(np.int64), ps.microbatches[p0:p1].copy(), int(ps.plan_ptr[p0]), \
        [b - a for a, b in ranges]
