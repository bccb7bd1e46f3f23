"""GPU parity of the training-label pipeline (§8(f) rows 2 and 4): dyo_trace_path (the execution
trace of a known control flow), dyo_partition (reading R18: the overlap partition and the L275
heuristics) and dyo_trainer (reading R19: SGD on the pilot), each against the oracle."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import workloads as WL
from oracle import afm as A, decode as D, partition as PT, train as TR, encode as E, pilot as Pm
from gpu_harness import make_ctx, F_NO_HOST_POOL


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()


def _op_index(wl):
    ops = []

    def rec(items):
        for it in items:
            if isinstance(it, WL.Op):
                ops.append(it)
            elif isinstance(it, WL.If):
                for br in it.branches:
                    rec(br)
            else:
                rec(it.body)
    rec(wl.program)
    return ops


def _same_path(wl, rows, ops, its):
    """The library's (operator, iteration) rows bound like the oracle's (R13) equal its rows."""
    idx = _op_index(wl)
    if len(rows) != len(ops):
        return False
    for r, o, k in zip(rows, ops, its):
        if (r is None) != (o < 0):
            return False
        if r is not None and A.bind(idx[o], int(k), 0) != r:
            return False
    return True


@pytest.mark.parametrize("name", ["tiny", "moe", "tree"])
def test_trace_path_matches_resolve(name):
    wl = WL.make(name, n_samples=4, **({"batch": 4} if name == "tree" else {}))
    d = make_ctx(wl, flags=F_NO_HOST_POOL, max_batch=4 if name == "tree" else 1)
    for s in range(3):
        ch = WL.actual_choices(wl, s)
        nested = []
        if name == "tree":
            nested = list(wl.notes["trees"][s])
            sl = A.sites(wl.program)
            ch = [len(nested) - sl[0].lo if i in (0, 2) else (-1 if c < 0 else c) for i, c in enumerate(ch)]
        rows = A.resolve(wl.program, [max(c, 0) for c in ch], 0, nested=nested or None)
        ops, its = d.trace_path([max(c, 0) for c in ch], nested)
        assert _same_path(wl, rows, ops.tolist(), its.tolist())
    d.close()


def _trace(wl, d, s):
    ch = [max(c, 0) for c in WL.actual_choices(wl, s)]
    rows = A.resolve(wl.program, ch, 0)
    ops, its = d.trace_path(ch)
    times = [WL.op_time_ns(r) for r in rows]
    op_ns = [WL.op_time_ns(o) for o in _op_index(wl)]
    return rows, times, ops, its, op_ns


def _wl(name):
    if name == "moe6":                        # 6 MoE layers: a trace short enough for the cubic oracle
        return WL.make_moe(n_samples=4, layers=6, layers_per_group=1, expert_mib=1, act_mib=1, budget=96 << 20)
    return WL.make(name, n_samples=4)


@pytest.mark.parametrize("name,K,H_frac,bw", [("tiny", 8, 0.5, 50_000), ("tiny", 4, 0.25, 5_000),
                                              ("moe6", 12, 1.0, 50_000), ("moe6", 6, 0.3, 2_000)])
def test_partition_matches_oracle(name, K, H_frac, bw):
    wl = _wl(name)
    d = make_ctx(wl, flags=F_NO_HOST_POOL)
    for s in range(2):
        rows, times, ops, its, op_ns = _trace(wl, d, s)
        need, fetch, comp = PT.block_tables(rows, times, wl.tensors, wl.align) if len(rows) <= 120 else (None, None, None)
        if need is None:
            pytest.skip("trace too long for the oracle's cubic tables")
        H = int(H_frac * sum(max(need[0][e] for e in range(1, len(rows) + 1)) for _ in [0]))
        want_cuts, want_ex = PT.overlap_partition(len(rows), K, need, fetch, comp, H, bw)
        cuts, ex, ok = d.partition(ops, its, 0, op_ns, K, "overlap", H, bw)
        if want_cuts is None:
            assert not ok and ex == -1
        else:
            assert ok and cuts == want_cuts and ex == want_ex
        for m, kind in ((1, "ops"), (2, "time"), (3, "size")):
            wc = PT.even_partition(PT.heuristic_weights(rows, times, wl.tensors, kind), K)
            c2, e2, ok2 = d.partition(ops, its, 0, op_ns, K, m, H, bw)
            assert c2 == wc and e2 == PT.exposed(wc, fetch, comp, bw) and ok2 == PT.feasible(wc, need, H)
    d.close()


@pytest.mark.parametrize("name,B,steps,lr", [("tiny", 8, 6, 0.01), ("moe", 16, 4, 1e-5)])
def test_trainer_matches_oracle_sgd(name, B, steps, lr):
    wl = WL.make(name, n_samples=max(16, B))
    spec = wl.pilot
    feats = np.stack([E.encode(wl, wl.samples[i], wl.hist_ids, ()) for i in range(B)])
    rng = np.random.default_rng(3)
    tgt = rng.uniform(-1, 1, size=(B, spec.O)).astype(np.float32)
    X = torch.from_numpy(feats.astype(np.float32)).cuda()
    T = torch.from_numpy(tgt).cuda()
    tr = __import__("paper_conf_hpca_renxyzlnwxl24_b200").Trainer(spec, wl.nn_type, B)
    w = TR.widen(spec)
    for k in range(steps):
        L_gpu = tr.step(X, T, B, lr=lr, stream=torch.cuda.current_stream().cuda_stream)
        L_or = TR.sgd_step(spec, w, feats.astype(np.float32).astype(np.float64), tgt.astype(np.float64), wl.nn_type, lr)
        assert abs(L_gpu - L_or) <= 1e-12 * max(1.0, abs(L_or)), (k, L_gpu, L_or)
    got = tr.weights()
    for name_ in TR.params(spec, wl.nn_type):
        err = np.abs(got[name_] - w[name_]).max()
        assert err <= 1e-12 * max(1.0, np.abs(w[name_]).max()), (name_, err)
    # untrained MLPs are returned unchanged
    other = (wl.nn_type + 1) % 3
    assert np.array_equal(got[f"mlp{other}.0.W"], spec.weights[f"mlp{other}.0.W"].astype(np.float64))
    tr.close()
