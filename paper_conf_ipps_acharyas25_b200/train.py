"""Training loop of the DAG-Transformer latency model.

The paper's recipe (SIV-B6-8): Adam with PyTorch defaults
(beta1 0.9, beta2 0.999), learning rate 1e-3 in the first epoch decayed by a
cosine to 0 in the last, up to 500 epochs of mini-batches of 32 stage graphs,
the MAE loss of Eqn 3, and early stopping: the weights of the best validation
loss are kept, and training stops (restoring them) once the validation loss
has not improved for 200 epochs.

Every step of the computation runs in libpredtop's kernels (predtop_train_grad
/ predtop_train_adam through predtop.Trainer); this module is host logic only:
the epoch loop, the learning-rate schedule, batch order and early stopping.
Reading R23: mini-batches are fixed partitions of the training
set (their DAGs are built once), visited in a seeded random order per epoch.
"""
from __future__ import annotations

import dataclasses
import math
from typing import List, Optional, Sequence, Tuple

import numpy as np
import torch

from . import predtop as pt


def cosine_lr(epoch: int, epochs: int, lr0: float = 1e-3) -> float:
    """lr0 in epoch 0, 0 in epoch epochs-1."""
    if epochs <= 1:
        return lr0
    return lr0 * 0.5 * (1.0 + math.cos(math.pi * epoch / (epochs - 1)))


@dataclasses.dataclass
class Batch:
    dag: "pt.Dag"
    y: torch.Tensor  # [G] fp32 device labels

    @property
    def num_graphs(self) -> int:
        return self.dag.batch.num_graphs


def make_batches(stage_batch, labels: np.ndarray, batch_size: int = 32, device="cuda") -> List[Batch]:
    """Split a synth.StageBatch (+ labels) into consecutive mini-batches with
    their DAGs built on the device (synchronous validation: training needs
    every graph valid)."""
    out = []
    G = stage_batch.num_graphs
    for lo in range(0, G, batch_size):
        idx = list(range(lo, min(G, lo + batch_size)))
        sub = stage_batch.subset(idx)
        dag = pt.Dag(pt.DeviceBatch.from_host(sub, device=device))
        if dag.status != pt.OK:
            raise pt.PredtopError(dag.status, f"invalid training graph {lo + dag.first_bad}")
        out.append(Batch(dag, torch.tensor(np.asarray(labels)[idx], dtype=torch.float32, device=device)))
    return out


def evaluate(trainer: "pt.Trainer", batches: Sequence[Batch]) -> float:
    """Mean absolute error over all graphs of the batches (fp32 training forward)."""
    tot, n = 0.0, 0
    for b in batches:
        loss, _ = trainer.grad(b.dag, b.y)
        tot += float(loss.item()) * b.num_graphs
        n += b.num_graphs
    return tot / max(n, 1)


@dataclasses.dataclass
class History:
    train: List[float]
    val: List[float]
    lr: List[float]
    best_epoch: int
    best_val: float
    stopped_early: bool


def train(trainer: "pt.Trainer", train_batches: Sequence[Batch], val_batches: Sequence[Batch], epochs: int = 500,
          lr0: float = 1e-3, patience: int = 200, seed: int = 0, log=None) -> History:
    """The paper's training loop; returns the history and leaves the best
    validation weights in the trainer."""
    rng = np.random.default_rng(seed)
    params = trainer.buffer(pt.Trainer.PARAMS)
    best = params.clone()
    best_val, best_epoch, since = float("inf"), -1, 0
    hist = History([], [], [], -1, float("inf"), False)
    for e in range(epochs):
        lr = cosine_lr(e, epochs, lr0)
        tot, n = 0.0, 0
        for i in rng.permutation(len(train_batches)):
            b = train_batches[i]
            loss, _ = trainer.grad(b.dag, b.y)
            trainer.adam(lr)
            tot += float(loss.item()) * b.num_graphs
            n += b.num_graphs
        val = evaluate(trainer, val_batches) if val_batches else tot / max(n, 1)
        hist.train.append(tot / max(n, 1))
        hist.val.append(val)
        hist.lr.append(lr)
        if val < best_val:
            best_val, best_epoch, since = val, e, 0
            best.copy_(params)
        else:
            since += 1
        if log:
            log(f"epoch {e:4d} lr {lr:.2e} train {hist.train[-1]:.5f} val {val:.5f} best {best_val:.5f}@{best_epoch}")
        if since >= patience:
            hist.stopped_early = True
            break
    params.copy_(best)
    hist.best_epoch, hist.best_val = best_epoch, best_val
    return hist
