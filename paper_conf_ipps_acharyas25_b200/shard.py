"""Multi-GPU plumbing of the prediction path.

Stage graphs are independent, and in owned mode a plan depends only on its own
stages, so the path shards by plans with no data-path exchange: each rank
scores a contiguous range of plans (and their stage graphs), then ONE
all-gather collects the fp64 plan latencies T on every rank, and every rank
takes the same argmin by (T, global plan id).  Only host-side index logic and
torch.distributed calls live here; the arithmetic runs in libpredtop.
"""
from __future__ import annotations

from typing import List, Sequence, Tuple

import numpy as np


def even_ranges(n: int, world: int) -> List[Tuple[int, int]]:
    """Split [0, n) into `world` contiguous ranges whose sizes differ by <= 1."""
    base, extra = divmod(n, world)
    out, s = [], 0
    for r in range(world):
        e = s + base + (1 if r < extra else 0)
        out.append((s, e))
        s = e
    return out


def balanced_ranges(costs: Sequence[float], world: int) -> List[Tuple[int, int]]:
    """Contiguous ranges of items with near-equal total cost (greedy on the
    prefix sum: range r ends where the prefix crosses (r+1)/world of the total).
    Used with the per-plan cost sum over its stages of (24 N d^2 + 4 d N^2)."""
    c = np.asarray(costs, np.float64)
    n = len(c)
    if n == 0:
        return [(0, 0)] * world
    pref = np.concatenate([[0.0], np.cumsum(c)])
    total = pref[-1]
    bounds = [0]
    for r in range(1, world):
        target = total * r / world
        k = int(np.searchsorted(pref, target, side="left"))
        k = min(max(k, bounds[-1]), n)
        bounds.append(k)
    bounds.append(n)
    return [(bounds[r], bounds[r + 1]) for r in range(world)]


def plan_costs(plan_ptr: np.ndarray, stage_nodes: np.ndarray, d: int) -> np.ndarray:
    """Estimated work per plan: sum over its stage graphs of 24 N d^2 + 4 d N^2
    (projections/FFN + attention with N^2 as the |A| proxy)."""
    n = np.asarray(stage_nodes, np.float64)
    per_stage = 24.0 * n * d * d + 4.0 * d * n * n
    pref = np.concatenate([[0.0], np.cumsum(per_stage)])
    pp = np.asarray(plan_ptr, np.int64)
    return pref[pp[1:]] - pref[pp[:-1]]


def gather_plan_latency(T_local, counts: Sequence[int], group=None):
    """All-gather variable-length fp64 plan latencies (rank r holds counts[r]
    plans, in global plan order r = 0..world-1).  Pads every shard to the max
    count with +inf for all_gather_into_tensor, then drops the padding.
    Works with NCCL (cuda tensors) and gloo (cpu tensors)."""
    import torch
    import torch.distributed as dist
    world = len(counts)
    m = max(counts) if counts else 0
    pad = torch.full((m,), float("inf"), dtype=torch.float64, device=T_local.device)
    pad[:T_local.numel()] = T_local
    out = torch.empty(world * m, dtype=torch.float64, device=T_local.device)
    if T_local.device.type == "cuda":
        dist.all_gather_into_tensor(out, pad, group=group)
    else:  # gloo has no all_gather_into_tensor on every build
        parts = [torch.empty_like(pad) for _ in range(world)]
        dist.all_gather(parts, pad, group=group)
        out = torch.cat(parts)
    if all(c == m for c in counts):
        return out
    keep = torch.cat([torch.arange(r * m, r * m + counts[r], device=out.device) for r in range(world)])
    return out[keep]


def argmin_by_T_then_id(T: np.ndarray) -> int:
    """Host reference of the ranking rule R13 (used by tests): smallest T,
    ties to the lower global plan id, NaN never chosen, all-NaN -> -1."""
    best = -1
    for i, v in enumerate(np.asarray(T, np.float64)):
        if np.isnan(v):
            continue
        if best < 0 or v < T[best]:
            best = i
    return best
