"""Pins for oracle/train.py (reading R19: SGD on the pilot)."""
import numpy as np

import workloads as WL
from oracle import train as TR


def _small_spec(seed=0, feature=True):
    rng = np.random.default_rng(seed)
    w = {}
    if feature:
        feat = [(0, 3, 4), (3, 5, 3), (8, 2, 2)]
        for i, (off, ln, out) in enumerate(feat):
            w[f"feat{i}.W"] = rng.normal(size=(out, ln))
            w[f"feat{i}.b"] = rng.normal(size=out)
        F, mlp = 16, [(9, 6), (6, 5)]
    else:
        feat, F, mlp = [], 16, [(16, 6), (6, 5)]
    for k in range(3):
        for l, (i, o) in enumerate(mlp):
            w[f"mlp{k}.{l}.W"] = rng.normal(size=(o, i))
            w[f"mlp{k}.{l}.b"] = rng.normal(size=o)
    w["out.W"] = rng.normal(size=(7, 5))
    w["out.b"] = rng.normal(size=7)
    return WL.PilotSpec(F=F, O=7, feature=feat, mlp=mlp, out_in=5, weights=w)


def test_gradients_match_central_differences():
    for feature in (True, False):
        spec = _small_spec(1, feature)
        w = TR.widen(spec)
        rng = np.random.default_rng(2)
        X = rng.normal(size=(4, 16))
        T = rng.normal(size=(4, 7))
        L, g = TR.loss_and_grads(spec, w, X, T, 1)
        h = 1e-6
        for name in TR.params(spec, 1):
            it = np.nditer(w[name], flags=["multi_index"])
            for _ in it:
                idx = it.multi_index
                w2 = {k: v.copy() for k, v in w.items()}
                w2[name][idx] += h
                Lp, _ = TR.loss_and_grads(spec, w2, X, T, 1)
                w2[name][idx] -= 2 * h
                Lm, _ = TR.loss_and_grads(spec, w2, X, T, 1)
                fd = (Lp - Lm) / (2 * h)
                assert abs(fd - g[name][idx]) <= 1e-6 * max(1.0, abs(fd)), (name, idx, fd, g[name][idx])


def test_lr_zero_and_unselected_mlps_unchanged():
    spec = _small_spec(3)
    w = TR.widen(spec)
    X = np.ones((2, 16))
    T = np.zeros((2, 7))
    w0 = {k: v.copy() for k, v in w.items()}
    TR.sgd_step(spec, w, X, T, 2, lr=0.0)
    assert all(np.array_equal(w[k], w0[k]) for k in w)
    TR.sgd_step(spec, w, X, T, 2, lr=0.01)
    for k in w:
        if k.startswith("mlp0.") or k.startswith("mlp1."):
            assert np.array_equal(w[k], w0[k])      # only the selected MLP runs
    assert not np.array_equal(w["out.b"], w0["out.b"])


def test_output_bias_step_closed_form():
    """dL/db_out = (2 / (B O)) sum over the batch of (y - t): one step moves the output bias by lr
    times that."""
    spec = _small_spec(4)
    w = TR.widen(spec)
    rng = np.random.default_rng(5)
    X, T = rng.normal(size=(3, 16)), rng.normal(size=(3, 7))
    y, _ = TR.forward(spec, w, X, 0)
    b0 = w["out.b"].copy()
    L = TR.sgd_step(spec, w, X, T, 0, lr=0.01)
    assert np.allclose(w["out.b"], b0 - 0.01 * 2 * (y - T).sum(axis=0) / (3 * 7), rtol=0, atol=1e-15)
    assert abs(L - ((y - T) ** 2).sum() / 21) <= 1e-12 * L


def test_sgd_decreases_loss_on_a_fixed_batch():
    spec = _small_spec(6)
    w = TR.widen(spec)
    rng = np.random.default_rng(7)
    X, T = rng.normal(size=(8, 16)), rng.normal(size=(8, 7))
    Ls = [TR.sgd_step(spec, w, X, T, 1, lr=0.01) for _ in range(50)]
    assert Ls[-1] < Ls[0]
