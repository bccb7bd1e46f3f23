"""Pilot-model forward pass in float64 (§IV-C, §V).

Oracle — test infrastructure only (see oracle/__init__.py).

Topology (reading R5): three input-feature layers (or an identity stage for the
tiny T32 pilot) -> the MLP selected by the NN type (only one of the three runs) ->
a linear output layer producing the logits. LeakyReLU with negative slope 0.01
(reading R5; the paper is silent) after every layer except the output layer.
"""
from __future__ import annotations

import numpy as np

SLOPE = 0.01


def leaky_relu(v):
    return np.where(v > 0, v, SLOPE * v)


def dense(Wt, b, x):
    """y = W x + b in float64 (W row-major [out][in])."""
    return Wt.astype(np.float64) @ x + b.astype(np.float64)


def forward(spec, x, nn_type):
    """Logits (float64) of one feature vector x (length F)."""
    w = spec.weights
    if spec.feature:
        parts = []
        for i, (off, ln, _o) in enumerate(spec.feature):
            parts.append(leaky_relu(dense(w[f"feat{i}.W"], w[f"feat{i}.b"], x[off:off + ln])))
        z = np.concatenate(parts)
    else:
        z = np.asarray(x, dtype=np.float64)
    k = int(nn_type)                      # the NN type activates one MLP
    for l in range(len(spec.mlp)):
        z = leaky_relu(dense(w[f"mlp{k}.{l}.W"], w[f"mlp{k}.{l}.b"], z))
    return dense(w["out.W"], w["out.b"], z)


def forward_abs(spec, x, nn_type):
    """Per-logit bound sum_k |w_ik||z_k| propagated layer by layer (for the fp32 error gate):
    returns (logits, mag) where mag_i = |b_i| + sum_k |W_ik| |z_k| of the output layer."""
    w = spec.weights
    if spec.feature:
        parts = []
        for i, (off, ln, _o) in enumerate(spec.feature):
            parts.append(leaky_relu(dense(w[f"feat{i}.W"], w[f"feat{i}.b"], x[off:off + ln])))
        z = np.concatenate(parts)
    else:
        z = np.asarray(x, dtype=np.float64)
    k = int(nn_type)
    for l in range(len(spec.mlp)):
        z = leaky_relu(dense(w[f"mlp{k}.{l}.W"], w[f"mlp{k}.{l}.b"], z))
    Wt, b = w["out.W"].astype(np.float64), w["out.b"].astype(np.float64)
    return Wt @ z + b, np.abs(Wt) @ np.abs(z) + np.abs(b)


def param_count(spec, active_only=False):
    n = 0
    for i, (off, ln, o) in enumerate(spec.feature):
        n += ln * o + o
    n_mlp = sum(i * o + o for i, o in spec.mlp)
    n += n_mlp if active_only else 3 * n_mlp
    n += spec.out_in * spec.O + spec.O
    return n
