"""GPU parity of the on-demand fetch of mis-predicted tensors (
DESIGN.md reading R17) through the C ABI: the harness plays the DyNN runtime - it migrates one
block ahead, asks dyo_fault_fetch for every access of the ACTUAL block (the actual path cut at
the predicted counts, oracle/fault.py), checks which accesses the library served from their
planned slot vs the fault area (oracle classification), reads every first-read tensor through
the returned address and compares its bytes with the latest version, writes new versions, and
at the end checks every host home and every resident device copy."""
import os
import subprocess
import sys

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import workloads as WL
from workloads import R, W
from oracle import plan as PL, fault as F, migrate as M
from gpu_harness import make_ctx, oracle_step, hist_for, tr_lists, gpu_lists

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()


class _Dev:
    def __init__(self, ptr, n):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": "|u1", "data": (ptr, False), "version": 3}


def _view(ptr, nb):
    return torch.as_tensor(_Dev(ptr, nb), device="cuda").view(torch.int32)


def _words(t, v, nb):
    return WL.content_words_torch(t, v, nb // 4, "cuda")


def run_faults(wl, steps, policy=1, drop=None, mispredict=False, area=256 << 20):
    d = make_ctx(wl, policy=policy)
    d.fault_config(area)
    pool = d.host_pool_array()
    for t, ten in enumerate(wl.tensors):
        pool[ten.host_off: ten.host_off + ten.nbytes] = M.content_bytes(t, 0, ten.nbytes)
    base, H = d.arena()
    stream = torch.cuda.current_stream()
    st = PL.initial_state(len(wl.tensors))
    table = ()
    ver = [0] * len(wl.tensors)
    n_fault = n_slot = 0
    hist = {}                                     # diagnostics: tensor -> [(step, block, kind, mode, planned)]
    for s in range(steps):
        smp = s % len(wl.samples)
        r = oracle_step(wl, [smp], st, table, policy, drop=drop)
        assert r["err"] is None
        pred = r["preds"][0]
        counts = [v[0] for v in pred.slots if v[0]]
        if mispredict:
            actual, _ = F.actual_sets(wl, WL.actual_choices(wl, smp), counts)
        else:
            actual = pred.W
        d.predict(wl.samples[[smp]].copy(), hist_for(wl, 1), 1, stream=stream.cuda_stream)
        K = d.plan(stream=stream.cuda_stream)
        assert K == len(r["trs"])
        fresh = set()
        for j, tr in enumerate(r["trs"]):
            assert gpu_lists(d, j) == tr_lists(tr)
            d.migrate(j, stream.cuda_stream)
            Aj = actual[j] if j < len(actual) else []
            cls = F.classify(r["Ws"][j], Aj)
            ptrs = d.fault_fetch(j, [t for t, _, _ in cls], [m for _, m, _ in cls], stream.cuda_stream)
            planned = {int(e[0]): int(e[3]) for e in d.plan_records(j, "entries").tolist()}
            pl = {t: (mm, rd) for t, mm, rd in r["Ws"][j]}
            for (t, m, kind), p in zip(cls, ptrs):
                hist.setdefault(t, []).append((s, j, kind, m, pl.get(t)))
            for t, mm, rd in r["Ws"][j]:
                if t not in {x for x, _, _ in cls}:
                    hist.setdefault(t, []).append((s, j, "planned-only", mm, rd))
            for (t, m, kind), p in zip(cls, ptrs):
                if kind == "slot":
                    assert p == base + planned[t], f"step {s} block {j}: tensor {t} not served from its slot"
                    n_slot += 1
                else:
                    assert not (base <= p < base + 2 * H), f"step {s} block {j}: tensor {t} should fault"
                    n_fault += 1
            # the actual block: first reads see the latest bytes, writes make new versions
            rd_first = {t for t, _, rd in Aj if rd}
            for (t, m, kind), p in zip(cls, ptrs):
                nb = wl.tensors[t].nbytes
                if t in rd_first and (not wl.tensors[t].transient or t in fresh):
                    assert torch.equal(_view(p, nb), _words(t, ver[t], nb)), f"step {s} block {j}: tensor {t} stale ({kind})"
            for (t, m, kind), p in zip(cls, ptrs):
                if m & W:
                    ver[t] += 1
                    fresh.add(t)
                    nb = wl.tensors[t].nbytes
                    _view(p, nb).copy_(_words(t, ver[t], nb))
        st, table = r["state"], r["table"]
    d.fault_flush(stream.cuda_stream)
    torch.cuda.synchronize()
    for t, ten in enumerate(wl.tensors):
        if ten.transient:
            continue
        if st.loc[t] != PL.HOST:
            got = _view(base + st.loc[t] * H + st.off[t], ten.nbytes)
            if not torch.equal(got, _words(t, ver[t], ten.nbytes)):
                have = [v for v in range(ver[t] + 1) if torch.equal(got, _words(t, v, ten.nbytes))]
                raise AssertionError(f"resident copy of {t} ({ten.name}): has version {have}, latest {ver[t]}; "
                                     f"history {hist.get(t)}")
        else:
            assert np.array_equal(pool[ten.host_off: ten.host_off + ten.nbytes], M.content_bytes(t, ver[t], ten.nbytes)), \
                f"host home of {t}"
    stats = d.fault_stats()
    d.close()
    assert stats["faults"] == n_fault and stats["resident"] == n_slot
    return n_fault, n_slot


def test_no_misprediction_serves_every_access_from_its_slot():
    wl = WL.make("tiny", n_samples=8)
    n_fault, n_slot = run_faults(wl, 3)
    assert n_fault == 0 and n_slot > 0


def test_injected_drops_fault_and_keep_bytes_exact():
    """DYO_FAULT-equivalent drops applied on the oracle side only would desynchronise the plans,
    so this case runs in a child process with DYO_FAULT set (read once per process)."""
    env = dict(os.environ, DYO_FAULT="drop_prefetch:0.3:7", PYTHONPATH=os.pathsep.join([ROOT, os.path.join(ROOT, "tests")]))
    code = ("import sys; sys.argv=['x']; import workloads as WL; from test_gpu_fault import run_faults; "
            "wl = WL.make('tiny', n_samples=8); wl.budget = 512 << 20; "
            "nf, ns = run_faults(wl, 4, drop=(0.3, 7)); assert nf > 0, nf; print('ok', nf, ns)")
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0 and "ok" in r.stdout, r.stdout[-3000:] + r.stderr[-3000:]


def test_mispredicted_routing_moe_scaled():
    """Natural mis-predictions: the actual routing (workloads.actual_choices, Zipf prior) differs
    from the pilot's; the other experts' weights fault in, gradients written by the actual
    backward blocks are written back (host home + device copy)."""
    wl = WL.make_moe(seed=2, n_samples=8, expert_mib=1, act_mib=1, budget=96 << 20)
    n_fault, n_slot = run_faults(wl, 4, mispredict=True, area=64 << 20)
    assert n_fault > 0 and n_slot > 0
