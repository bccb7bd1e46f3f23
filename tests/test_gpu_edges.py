"""GPU parity on degenerate and ragged inputs (survey §8(c), ③ edge cases): an all-zero output
layer (empty block head -> one group over the whole path, R4; all-tied branch logits -> lowest
index), ragged tensor-core batches (B not a multiple of the 64-sample tile), batch 1 on a ctx
sized for 64, and a plan of the degenerate predictions."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import workloads as WL
from oracle import plan as PL
from gpu_harness import make_ctx, oracle_step, hist_for, tr_lists, gpu_lists, F_NO_HOST_POOL
from test_gpu_parity import _check_prediction, _stream


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()


def _zero_output(wl):
    w = wl.pilot.weights
    for k in list(w):
        if k.startswith("out."):
            w[k] = np.zeros_like(w[k])
    return wl


@pytest.mark.parametrize("name,B", [("tiny", 1), ("tiny", 4), ("moe", 1), ("moe", 20)])
def test_zero_output_layer_one_group(name, B):
    wl = _zero_output(WL.make(name, n_samples=max(16, B)))
    d = make_ctx(wl, max_batch=B, flags=F_NO_HOST_POOL)
    d.predict(wl.samples[:B].copy(), hist_for(wl, B), B, stream=_stream())
    r = oracle_step(wl, range(B), PL.initial_state(len(wl.tensors)), ())
    for b in range(B):
        p = r["preds"][b]
        assert len(p.groups) == 1 and p.groups[0] == (0, len(p.path))     # R4: no non-empty slot
        assert all(c == 0 or s.tie >= 0 for c, s in zip(p.choices, __import__("oracle").afm.sites(wl.program)))
        _check_prediction(d, wl, b, p)
    if r["err"] is None:
        K = d.plan(stream=_stream())
        assert K == len(r["trs"])
        for j, tr in enumerate(r["trs"]):
            assert gpu_lists(d, j) == tr_lists(tr)
    d.close()


@pytest.mark.parametrize("name,B", [("moe", 17), ("moe", 63), ("lstm", 33)])
def test_ragged_tensor_core_batches(name, B):
    wl = WL.make(name, n_samples=max(16, B + 1))
    d = make_ctx(wl, max_batch=64, flags=F_NO_HOST_POOL)
    d.predict(wl.samples[:B].copy(), hist_for(wl, B), B, stream=_stream())
    r = oracle_step(wl, range(B), PL.initial_state(len(wl.tensors)), (), plan=False)
    for b in range(B):
        _check_prediction(d, wl, b, r["preds"][b])
    # then a batch of one on the same ctx (the cluster GEMV path)
    d.predict(wl.samples[B:B + 1].copy(), hist_for(wl, 1), 1, stream=_stream())
    r1 = oracle_step(wl, [B], PL.initial_state(len(wl.tensors)), r["table"], plan=False)
    _check_prediction(d, wl, 0, r1["preds"][0])
    d.close()


def test_max_batch_1024_predict_and_plan():
    """Maximum sizes: the largest prediction batch the ABI accepts (max_batch 1024) on the tiny
    workload - 1,024 predictions in one dyo_pilot_predict (batch kernel, clusters co-resident by
    the launch's cluster-size choice), decoded on the GPU, then one plan of their 8,192 groups:
    logits (north_star gate) and decodes on a sample of the predictions, every transition of the
    plan bit-exact with the oracle."""
    from gpu_harness import logit_gates
    B = 1024
    wl = WL.make("tiny", n_samples=B)
    d = make_ctx(wl, max_batch=B, flags=F_NO_HOST_POOL)
    logits = torch.zeros((B, wl.pilot.O), device="cuda")
    d.predict(wl.samples[:B].copy(), hist_for(wl, B), B, logits, stream=_stream())
    r = oracle_step(wl, range(B), PL.initial_state(len(wl.tensors)), ())
    assert r["err"] is None
    y = logits.cpu().numpy()
    for b in list(range(0, B, 97)) + [B - 1]:
        g1, g2, _ = logit_gates(y[b], r["feats"][b], wl.pilot, wl.nn_type)
        assert g1.all() and g2.all(), f"prediction {b}"
        _check_prediction(d, wl, b, r["preds"][b])
    K = d.plan(stream=_stream())
    assert K == len(r["trs"]) == sum(len(p.W) for p in r["preds"])
    for j, tr in enumerate(r["trs"]):
        info = d.plan_info(j)
        assert (info["half"], info["h2d"], info["d2h"], info["d2d"], info["need"]) == \
            (tr.half, tr.h2d, tr.d2h, tr.d2d, tr.need), f"transition {j}"
        assert gpu_lists(d, j) == tr_lists(tr), f"transition {j}"
    d.close()
