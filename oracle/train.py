"""Pilot training (§IV-D "a pilot-training sample is a pair of an input vector and an
output vector"; §V "LeakyReLU as activation, SGD as optimizer, and 0.01 as learning rate";
DESIGN.md reading R19).

Oracle - test infrastructure only (see oracle/__init__.py).

Loss (reading R19; the paper names no loss): for a minibatch of B samples with pilot outputs y_b
(O logits each) and targets t_b (the label block vectors in the block-head units of R4 - count /
16, idiom sums / 16, dimension sums / 1024 - and, in the branch head, the one-hot of each free
site's actual choice), the mean squared error L = (1 / (B O)) sum_b ||y_b - t_b||^2 (PyTorch's
MSELoss default reduction). One SGD step: every parameter p <- p - lr dL/dp,
where the parameters are the feature layers, the MLP selected by the NN type (the only one that
runs) and the output layer. fp64 throughout (the pilot's fp32 weights are widened
exactly; a trained pilot is rounded back to fp32 to be loaded).
"""
from __future__ import annotations

import numpy as np

SLOPE = 0.01


def params(spec, nn_type):
    """Names of the trained parameters in update order."""
    names = []
    for i in range(len(spec.feature)):
        names += [f"feat{i}.W", f"feat{i}.b"]
    for l in range(len(spec.mlp)):
        names += [f"mlp{nn_type}.{l}.W", f"mlp{nn_type}.{l}.b"]
    return names + ["out.W", "out.b"]


def forward(spec, w, X, nn_type):
    """Minibatch forward (X: B x F float64). Returns the output and the cache of every layer's
    input and post-activation for the backward pass."""
    cache = []
    if spec.feature:
        outs = []
        for i, (off, ln, _) in enumerate(spec.feature):
            z = X[:, off:off + ln]
            v = z @ w[f"feat{i}.W"].T + w[f"feat{i}.b"]
            a = np.where(v > 0, v, SLOPE * v)
            cache.append((f"feat{i}", z, a))
            outs.append(a)
        h = np.concatenate(outs, axis=1)
    else:
        h = X
    for l in range(len(spec.mlp)):
        v = h @ w[f"mlp{nn_type}.{l}.W"].T + w[f"mlp{nn_type}.{l}.b"]
        a = np.where(v > 0, v, SLOPE * v)
        cache.append((f"mlp{nn_type}.{l}", h, a))
        h = a
    y = h @ w["out.W"].T + w["out.b"]
    cache.append(("out", h, None))
    return y, cache


def loss_and_grads(spec, w, X, Tgt, nn_type):
    """(L, {name: dL/dname}) by backpropagation through the cache."""
    B = X.shape[0]
    y, cache = forward(spec, w, X, nn_type)
    diff = y - Tgt
    N = diff.size
    L = float((diff * diff).sum() / N)
    g = {}
    d = 2.0 * diff / N                             # dL/dy
    # output layer (linear)
    name, z, _ = cache[-1]
    g["out.W"] = d.T @ z
    g["out.b"] = d.sum(axis=0)
    dh = d @ w["out.W"]
    # MLP layers, last to first
    n_mlp = len(spec.mlp)
    for l in range(n_mlp - 1, -1, -1):
        name, z, a = cache[len(cache) - 1 - (n_mlp - l)]
        dv = dh * np.where(a > 0, 1.0, SLOPE)
        g[f"{name}.W"] = dv.T @ z
        g[f"{name}.b"] = dv.sum(axis=0)
        dh = dv @ w[f"{name}.W"]
    # feature layers: dh is the gradient w.r.t. their concatenated outputs
    if spec.feature:
        o = 0
        for i, (off, ln, out) in enumerate(spec.feature):
            name, z, a = cache[i]
            dv = dh[:, o:o + out] * np.where(a > 0, 1.0, SLOPE)
            g[f"{name}.W"] = dv.T @ z
            g[f"{name}.b"] = dv.sum(axis=0)
            o += out
    return L, g


def sgd_step(spec, w, X, Tgt, nn_type, lr=0.01):
    """One SGD step in place on the float64 weights w; returns the loss before the step."""
    L, g = loss_and_grads(spec, w, X, Tgt, nn_type)
    for name in params(spec, nn_type):
        w[name] = w[name] - lr * g[name]
    return L


def widen(spec):
    return {k: np.asarray(v, np.float64).copy() for k, v in spec.weights.items()}


def targets(wl, label_blocks, choices, O):
    """Pilot-output targets of one sample (R19): the label block vectors in R4's block-head units
    (elements 0..6 / 16, 7..9 / 1024), then the branch head: one-hot of each free top-level
    site's choice; zeros elsewhere."""
    from . import afm as A
    t = np.zeros(O, np.float64)
    for k, v in enumerate(label_blocks):
        for e in range(10):
            t[10 * k + e] = v[e] / (16.0 if e < 7 else 1024.0)
    off = 10 * wl.K_max
    sl = A.sites(wl.program)
    inner = A.nested_ids(wl.program)
    for i, s in enumerate(sl):
        if id(s) in inner or s.tie >= 0:
            continue
        t[off + choices[i]] = 1.0
        off += A.n_choices(s)
    return t
