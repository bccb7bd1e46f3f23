"""Pins for oracle/pilot.py: closed forms, textbook MLP (torch.nn), MLP selection invariance."""
import copy

import numpy as np
import pytest
import torch

from oracle import pilot as P
import workloads as WL


@pytest.mark.parametrize("name", ["tiny", "moe"])
def test_zero_weights_give_output_bias(name):
    wl = WL.make(name)
    spec = copy.deepcopy(wl.pilot)
    for k in spec.weights:
        spec.weights[k] = np.zeros_like(spec.weights[k])
    spec.weights["out.b"] = np.arange(spec.O, dtype=np.float32) - 7
    y = P.forward(spec, np.ones(spec.F), wl.nn_type)
    assert np.array_equal(y, spec.weights["out.b"].astype(np.float64))


def test_positive_case_is_affine_chain():
    """All-positive weights, biases and inputs: LeakyReLU is the identity, so the pilot is the
    composition of affine maps; compare with the composed matrix applied once."""
    rng = np.random.default_rng(1)
    wl = WL.make("tiny")
    spec = copy.deepcopy(wl.pilot)
    for k in spec.weights:
        spec.weights[k] = rng.uniform(0, 0.1, spec.weights[k].shape).astype(np.float32)
    x = rng.uniform(0, 1, spec.F)
    k = wl.nn_type
    Wc = np.eye(spec.F)
    bc = np.zeros(spec.F)
    for l in range(len(spec.mlp)):
        Wl = spec.weights[f"mlp{k}.{l}.W"].astype(np.float64)
        bl = spec.weights[f"mlp{k}.{l}.b"].astype(np.float64)
        Wc, bc = Wl @ Wc, Wl @ bc + bl
    Wo = spec.weights["out.W"].astype(np.float64)
    want = Wo @ (Wc @ x + bc) + spec.weights["out.b"].astype(np.float64)
    np.testing.assert_allclose(P.forward(spec, x, k), want, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("name", ["tiny", "moe"])
def test_matches_torch_nn_modules(name):
    """The topology of P:L155-L158 written with torch.nn (float64) as a textbook reference."""
    wl = WL.make(name)
    spec = wl.pilot
    w = {k: torch.tensor(v, dtype=torch.float64) for k, v in spec.weights.items()}
    act = torch.nn.LeakyReLU(0.01)

    def lin(prefix):
        m = torch.nn.Linear(w[prefix + ".W"].shape[1], w[prefix + ".W"].shape[0]).double()
        with torch.no_grad():
            m.weight.copy_(w[prefix + ".W"])
            m.bias.copy_(w[prefix + ".b"])
        return m
    for s in range(3):
        x = torch.tensor(__import__("oracle.encode", fromlist=["x"]).encode(wl, wl.samples[s], wl.hist_ids, ()))
        if spec.feature:
            z = torch.cat([act(lin(f"feat{i}")(x[off:off + ln])) for i, (off, ln, _) in enumerate(spec.feature)])
        else:
            z = x
        mlp = torch.nn.Sequential(*[m for l in range(len(spec.mlp)) for m in (lin(f"mlp{wl.nn_type}.{l}"), act)])
        y = lin("out")(mlp(z)).detach().numpy()
        np.testing.assert_allclose(P.forward(spec, x.numpy(), wl.nn_type), y, rtol=1e-12, atol=1e-9)


def test_unselected_mlps_do_not_matter():
    wl = WL.make("moe")
    x = np.random.default_rng(0).uniform(-1, 1, wl.pilot.F)
    y0 = P.forward(wl.pilot, x, wl.nn_type)
    spec = copy.deepcopy(wl.pilot)
    for k in range(3):
        if k != wl.nn_type:
            for l in range(len(spec.mlp)):
                spec.weights[f"mlp{k}.{l}.W"] += 1.0
    assert np.array_equal(P.forward(spec, x, wl.nn_type), y0)
    spec.weights[f"mlp{wl.nn_type}.0.b"] += 1.0
    assert not np.array_equal(P.forward(spec, x, wl.nn_type), y0)


def test_leaky_slope():
    assert P.leaky_relu(np.array([-2.0, 3.0])).tolist() == [-0.02, 3.0]


def test_param_counts():
    wl = WL.make("tiny")       # T32: F=64 -> 32 -> 32, output 32 -> 88
    assert P.param_count(wl.pilot) == 3 * (64 * 32 + 32 + 32 * 32 + 32) + 32 * 88 + 88
    moe = WL.make("moe")       # P512: feature 16->32, 180->32, 3->32; MLP 96-512-512-512-64; out 64->544
    feat = 16 * 32 + 32 + 180 * 32 + 32 + 3 * 32 + 32
    mlp = 96 * 512 + 512 + 2 * (512 * 512 + 512) + 512 * 64 + 64
    assert P.param_count(moe.pilot, active_only=True) == feat + mlp + 64 * 544 + 544
