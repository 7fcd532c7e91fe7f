"""Shared stage table + plan search (R20).

PredTOP's prediction phase: "we select all the stages for prediction
... After we get the latencies of all the stages on all different meshes we
use the pipeline model to get the end-to-end latency".  Alpa enumerates every
stage = contiguous layer range on every mesh; PredTOP trains one
model per mesh configuration (Tables II-III).  One step here:

  1. predtop_build_dag over this rank's stage DAGs (a contiguous, cost-balanced
     range of the L(L+1)/2 layer-range stages, in packed-triangle order);
  2. predtop_stage_forward once per mesh choice c, writing the latencies
     straight into row c of the stage table [K][L(L+1)/2] (the table layout
     of predtop_plan_search, so no reshuffle);
  3. multi-GPU: ONE all-reduce (sum) of the table: every rank contributes its
     own range and zeros elsewhere, so the sum is exact and every rank holds
     the whole table (collective 1 of the two-collective variant);
  4. predtop_plan_search for every microbatch count B of interest (problems
     share the table), replicated on every rank: bitwise identical results,
     so no second collective is needed.

Host code only marshals; every arithmetic step runs in libpredtop.
"""
from __future__ import annotations

from typing import List, Sequence

import numpy as np


def stage_costs(sizes: Sequence[int], d: int) -> np.ndarray:
    n = np.asarray(sizes, np.float64)
    return 24.0 * n * d * d + 4.0 * d * n * n


class StageTableSearch:
    def __init__(self, pt, cfgs: List[dict], blobs: List[np.ndarray], batch, num_layers: int,
                 choice_devices: Sequence[int], num_devices: int, microbatches: Sequence[int],
                 rank: int = 0, world: int = 1, group=None, device="cuda", hops: int = 0):
        import torch
        from . import shard
        self.pt, self.torch = pt, torch
        self.L, self.K = int(num_layers), len(choice_devices)
        self.NT = self.L * (self.L + 1) // 2
        assert batch.num_graphs == self.NT, "batch must hold every layer-range stage in tri order"
        assert len(cfgs) == self.K == len(blobs)
        self.rank, self.world, self.group = rank, world, group
        self.ranges = shard.balanced_ranges(stage_costs(batch.sizes, cfgs[0]["d_model"]), world)
        self.g0, self.g1 = self.ranges[rank]
        self.models = [pt.Model(c, b, device=device) for c, b in zip(cfgs, blobs)]
        self.local = batch.subset(range(self.g0, self.g1)) if self.g1 > self.g0 else None
        self.db = pt.DeviceBatch.from_host(self.local, device=device) if self.local is not None else None
        self.dag = pt.Dag(self.db, no_sync=True, hops=hops) if self.db is not None else None
        self.ws = max((m.forward_workspace(self.dag) for m in self.models), key=lambda t: t.numel()) \
            if self.dag is not None else None
        # row c of `table` is the stage table of choice c; ranks write their own range
        self.table = torch.zeros((1, self.K, self.NT), dtype=torch.float32, device=device)
        self.mine = torch.zeros_like(self.table) if world > 1 else self.table
        self.B = torch.tensor(list(microbatches), dtype=torch.int32, device=device)
        self.table_of = torch.zeros(len(microbatches), dtype=torch.int32, device=device)  # one shared table
        self.search = pt.PlanSearch(len(microbatches), self.L, choice_devices, num_devices, device=device)

    def score(self):
        """Steps 1-2: this rank's stage DAGs on every mesh model -> its table range."""
        if self.dag is None:
            return
        self.dag.rebuild()
        for c, m in enumerate(self.models):
            m.forward(self.dag, workspace=self.ws, out=self.mine[0, c, self.g0:self.g1])

    def gather(self):
        """Step 3 (multi-GPU): the exact sum-all-reduce of disjoint ranges
        (NCCL on the device tensor; a host round trip for gloo)."""
        if self.world > 1:
            import torch.distributed as dist
            if dist.get_backend(self.group) == "gloo":
                t = self.mine.cpu()
                dist.all_reduce(t, group=self.group)
                self.table.copy_(t)
            else:
                self.table.copy_(self.mine)
                dist.all_reduce(self.table, group=self.group)

    def step(self):
        self.score()
        self.gather()
        return self.search.run(self.table, self.B, self.table_of)

    @property
    def graphs_local(self) -> int:
        return self.g1 - self.g0


def assemble_table_host(parts, K: int, NT: int):
    """Host reference of step 3 (tests): ranks' (g0, g1, rows [K][g1-g0]) ->
    the full [K][NT] table."""
    t = np.zeros((K, NT), np.float32)
    for g0, g1, rows in parts:
        t[:, g0:g1] = rows
    return t
