"""The compiled single-core CPU planner (baseline/cpu_planner.cpp, the bench's honest baseline for
K2) is bit-exact with oracle/plan.py."""
import sys
import os

import pytest

import workloads as WL
from oracle import plan as PL
from gpu_harness import oracle_step, tr_lists

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "baseline"))


@pytest.fixture(scope="module")
def planner():
    import __graft_entry__
    __graft_entry__.build()
    import cpu_planner
    return cpu_planner


@pytest.mark.parametrize("name,steps,B,policy,kw", [
    ("tiny", 6, 1, 1, {}), ("tiny", 6, 1, 0, {}), ("moe", 3, 1, 1, {}), ("tiny", 6, 1, 3, {}), ("af", 1, 1, 3, {}),
    ("lstm", 2, 8, 3, {"batch": 8, "max_len": 96, "n_samples": 32}),
    ("lstm", 2, 8, 1, {"batch": 8, "max_len": 96, "n_samples": 32}),
    ("tree", 2, 8, 1, {"batch": 8, "max_leaves": 24, "budget": 64 << 20, "n_samples": 32})])
def test_cpu_planner_bitexact(planner, name, steps, B, policy, kw):
    kw = dict(kw)
    n = kw.pop("n_samples", 32)
    wl = WL.make(name, n_samples=n, **kw)
    if name == "tiny":
        wl.budget = 384 << 20
    cp = planner.CpuPlanner(wl, policy)
    st, table = PL.initial_state(len(wl.tensors)), ()
    for s in range(steps):
        ids = [(s * B + i) % n for i in range(B)]
        r = oracle_step(wl, ids, st, table, policy)
        status, trs = cp.plan(r["Ws"])
        if r["err"] is not None:
            assert status == -3
            continue
        assert status == 0 and len(trs) == len(r["trs"])
        for j, tr in enumerate(r["trs"]):
            got = {k: trs[j][k] for k in ("evict", "move", "carry", "alloc", "fetch")}
            assert got == tr_lists(tr), f"step {s} transition {j}"
            assert (trs[j]["half"], trs[j]["h2d"], trs[j]["d2h"], trs[j]["d2d"], trs[j]["need"]) == \
                (tr.half, tr.h2d, tr.d2h, tr.d2d, tr.need)
        st, table = r["state"], r["table"]
    cp.close()
