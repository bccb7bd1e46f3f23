"""Host logic of bench.py's step bounds (no GPU): the record-level DAG (R21 / R12) and its
link-aware fluid model. Properties: the fluid model with an unlimited bidirectional aggregate is
the DAG bound; a finite aggregate can only lengthen it; the strict order is never shorter than the
per-range order; a single direction's bytes at its rate bound everything from below."""
import importlib.util
import os

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def bench():
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def _trace(rng, K=12):
    trs = []
    for j in range(K):
        wb = [(int(rng.integers(0, 64)) << 20, int(rng.integers(1, 32)) << 20) for _ in range(int(rng.integers(0, 4)))]
        fe = [(int(rng.integers(0, 64)) << 20, int(rng.integers(1, 32)) << 20) for _ in range(int(rng.integers(0, 4)))]
        trs.append((sum(n for _, n in fe), sum(n for _, n in wb), wb, fe, int(rng.integers(0, 2)) * int(rng.integers(0, 3)),
                    False, bool(rng.integers(0, 2))))
    return trs


@pytest.mark.parametrize("seed", range(20))
def test_bound_properties(bench, seed):
    trs = _trace(np.random.default_rng(seed))
    rh, rd = 55.0, 57.0
    dag = bench.step_bound_ms(trs, rh, rd)
    strict = bench.step_bound_ms(trs, rh, rd, strict=True)
    assert strict >= dag - 1e-9
    assert bench.step_bound_fluid_ms(trs, rh, rd, 1e12) == pytest.approx(dag, rel=1e-9, abs=1e-9)
    assert bench.step_bound_fluid_ms(trs, rh, rd, 90.0) >= dag - 1e-9
    lower = max(sum(t[0] for t in trs) / (rh * 1e6), sum(t[1] for t in trs) / (rd * 1e6))
    assert dag >= lower - 1e-9


def test_bound_hand_case(bench):
    """One transition: 50 MB written back, then a 60 MB fetch into that range and a 40 MB fetch
    elsewhere. Strict: 50/57 + 100/55 ms. Per-range (R21): the 40 MB fetch cannot overtake the
    first (the copy stream is in order), so the first waits for the write-back: same total; with
    the fetches in the other order the 40 MB one runs under the write-back."""
    wb = [(0, 50_000_000)]
    t1 = [(100e6, 50e6, wb, [(0, 60_000_000), (100_000_000, 40_000_000)], 0, False, False)]
    t2 = [(100e6, 50e6, wb, [(100_000_000, 40_000_000), (0, 60_000_000)], 0, False, False)]
    s = 50e6 / 57e6 + 100e6 / 55e6
    assert bench.step_bound_ms(t1, 55.0, 57.0, strict=True) == pytest.approx(s)
    assert bench.step_bound_ms(t1, 55.0, 57.0) == pytest.approx(s)
    assert bench.step_bound_ms(t2, 55.0, 57.0) == pytest.approx(max(40e6 / 55e6, 50e6 / 57e6) + 60e6 / 55e6)
