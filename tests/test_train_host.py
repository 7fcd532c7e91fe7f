"""Host logic of the training loop (paper_conf_ipps_acharyas25_b200/train.py)
without a GPU: the cosine schedule, the seeded batch order, and early
stopping with best-weight restore, driven by a scripted stand-in for
predtop.Trainer (the kernels themselves are covered by tests/test_gpu_train.py)."""
import types

import numpy as np
import pytest
import torch

from paper_conf_ipps_acharyas25_b200 import train


class FakeTrainer:
    PARAMS = 0

    def __init__(self, val_curve):
        self.params = torch.zeros(4)
        self.val_curve = list(val_curve)
        self.lrs = []
        self.mode_val = False

    def buffer(self, which):
        return self.params

    def grad(self, dag, y):
        if dag.kind == "val":
            v = self.val_curve[min(len(self.lrs) // 2 - 1, len(self.val_curve) - 1)]
            return torch.tensor([v]), None
        return torch.tensor([1.0]), None

    def adam(self, lr):
        self.lrs.append(lr)
        self.params += 1.0  # parameters move every step: the epoch count is readable from them


def _batches(kind, n):
    return [train.Batch(types.SimpleNamespace(kind=kind, batch=types.SimpleNamespace(num_graphs=32)),
                        torch.zeros(32)) for _ in range(n)]


def test_cosine_schedule():
    E = 501
    lrs = [train.cosine_lr(e, E) for e in range(E)]
    assert lrs[0] == 1e-3 and abs(lrs[-1]) < 1e-15
    assert all(a >= b for a, b in zip(lrs, lrs[1:]))
    assert lrs[(E - 1) // 2] == pytest.approx(5e-4, rel=1e-12)


def test_early_stopping_restores_best():
    # validation: improves until epoch 3 (0.2), then never again
    curve = [1.0, 0.5, 0.3, 0.2] + [0.4] * 50
    tr = FakeTrainer(curve)
    hist = train.train(tr, _batches("train", 2), _batches("val", 1), epochs=100, patience=5, seed=1)
    assert hist.best_epoch == 3 and hist.best_val == pytest.approx(0.2)
    assert hist.stopped_early and len(hist.val) == 3 + 1 + 5
    # best weights = after epoch 3 = 4 epochs x 2 steps of +1
    assert torch.equal(tr.params, torch.full((4,), 8.0))
    assert len(tr.lrs) == 2 * len(hist.val)
    np.testing.assert_allclose(tr.lrs[::2], [train.cosine_lr(e, 100) for e in range(len(hist.val))])


def test_no_early_stop_runs_all_epochs():
    curve = list(np.linspace(1.0, 0.1, 12))
    tr = FakeTrainer(curve)
    hist = train.train(tr, _batches("train", 2), _batches("val", 1), epochs=12, patience=200, seed=0)
    assert not hist.stopped_early and len(hist.val) == 12 and hist.best_epoch == 11
