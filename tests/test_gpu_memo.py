"""GPU parity of the mis-prediction record + exact-match memo (reading
R15) through the C ABI: reported mis-predictions, memo hits taken inside the decode kernels
(fused pilot epilogue, stand-alone head kernel, tensor-core batch path) and the memo-resolved
predictions element by element against oracle/memo.py."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import workloads as WL
from oracle import memo as M, plan as PL
from gpu_harness import make_ctx, oracle_step, F_NO_HOST_POOL
from test_gpu_parity import _check_prediction, _stream


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()


@pytest.mark.parametrize("name,B", [("tiny", 1), ("tiny", 8), ("moe", 1), ("moe", 16), ("moe", 64), ("af", 2)])
def test_memo_parity(name, B):
    wl = WL.make(name, n_samples=max(16, B))
    d = make_ctx(wl, max_batch=B, flags=F_NO_HOST_POOL)
    d.memo_config(256)
    m = M.Memo(256)
    ids = list(range(B))
    samples = wl.samples[ids].copy()
    # pass 1: no memo entries; every prediction is the pilot's own (history-free features)
    d.predict(samples, None, B, stream=_stream())
    r = oracle_step(wl, ids, PL.initial_state(len(wl.tensors)), (), plan=False)
    n_bad = 0
    for b in range(B):
        _check_prediction(d, wl, b, r["preds"][b])
        act = WL.actual_choices(wl, ids[b])
        got = d.report(b, act)
        assert got == m.report(r["preds"][b], act, sample=ids[b])
        n_bad += int(got)
    assert n_bad > 0, "the seeded samples must contain mis-predictions"
    st = d.memo_stats()
    assert st["mispredictions"] == m.mispredictions and st["live"] == len(m.table)
    # pass 2: the same outputs hit the memo and resolve the actual control flow
    d.predict(samples, None, B, stream=_stream())
    hits = 0
    for b in range(B):
        exp, hit = M.decode_with_memo(wl, r["logits"][b], m, b=b)
        hits += int(hit)
        _check_prediction(d, wl, b, exp)
        # a memo-resolved prediction is no longer a mis-prediction of the reported flow
        if hit and tuple(exp.choices) == tuple(WL.actual_choices(wl, ids[b])):
            assert d.report(b, WL.actual_choices(wl, ids[b])) is False
    assert hits > 0
    assert d.memo_stats()["hits"] == hits
    d.close()


def test_memo_capacity_and_validation():
    wl = WL.make("tiny", n_samples=16)
    d = make_ctx(wl, max_batch=8, flags=F_NO_HOST_POOL)
    d.memo_config(1)
    m = M.Memo(1)
    ids = list(range(8))
    d.predict(wl.samples[ids].copy(), None, 8, stream=_stream())
    r = oracle_step(wl, ids, PL.initial_state(len(wl.tensors)), (), plan=False)
    for b in range(8):
        act = WL.actual_choices(wl, b)
        assert d.report(b, act) == m.report(r["preds"][b], act)
    assert d.memo_stats()["live"] == len(m.table) <= 1
    d.predict(wl.samples[ids].copy(), None, 8, stream=_stream())
    for b in range(8):
        exp, _ = M.decode_with_memo(wl, r["logits"][b], m, b=b)
        _check_prediction(d, wl, b, exp)
    # invalid reports: out-of-range choice, tie violation (R6), bad prediction index
    from paper_conf_hpca_renxyzlnwxl24_b200.dyo import DyoError
    with pytest.raises(DyoError):
        d.report(0, [5, 0, 0])
    with pytest.raises(DyoError):
        d.report(99, WL.actual_choices(wl, 0))
    d.close()
    wm = WL.make("moe", n_samples=2)
    dm = make_ctx(wm, max_batch=1, flags=F_NO_HOST_POOL)
    dm.predict(wm.samples[:1].copy(), None, 1, stream=_stream())
    from oracle import afm as A
    sl = A.sites(wm.program)
    bad = list(WL.actual_choices(wm, 0))
    tied = next(i for i, s in enumerate(sl) if s.tie >= 0)
    bad[tied] = (bad[tied] + 1) % A.n_choices(sl[tied])
    with pytest.raises(DyoError):
        dm.report(0, bad)
    dm.close()
