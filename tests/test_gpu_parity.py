"""GPU parity: libdyo (through its C ABI) against the CPU oracle, element by element."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import workloads as WL
from oracle import plan as PL, afm as A
from gpu_harness import (make_ctx, oracle_step, hist_for, tr_lists, gpu_lists, logit_gates,
                         F_NO_HOST_POOL, F_PILOT_TC)


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()


def _stream():
    return torch.cuda.current_stream().cuda_stream


@pytest.mark.parametrize("name", ["tiny", "moe", "af"])
def test_encode_bitexact(name):
    wl = WL.make(name)
    B = 4
    d = make_ctx(wl, max_batch=B, flags=F_NO_HOST_POOL)
    feat = torch.zeros((B, wl.pilot.F), device="cuda")
    d.encode(wl.samples[:B].copy(), hist_for(wl, B), B, feat, _stream())
    r = oracle_step(wl, range(B), PL.initial_state(len(wl.tensors)), ())
    got = feat.cpu().numpy().astype(np.float64)
    assert np.array_equal(got, np.stack(r["feats"]))
    # after a prediction the history table is the executed block vectors (R3)
    d.predict(wl.samples[:B].copy(), hist_for(wl, B), B, stream=_stream())
    d.encode(wl.samples[B:2 * B].copy(), hist_for(wl, B), B, feat, _stream())
    r2 = oracle_step(wl, range(B, 2 * B), PL.initial_state(len(wl.tensors)), r["table"])
    assert np.array_equal(feat.cpu().numpy().astype(np.float64), np.stack(r2["feats"]))
    d.close()


@pytest.mark.parametrize("name,B", [("tiny", 1), ("tiny", 16), ("moe", 1), ("moe", 8), ("af", 1), ("af", 3),
                                    ("lstm", 8), ("lstm", 64), ("moe", 64), ("af", 64), ("moe", 20), ("moe", 100),
                                    ("af", 17), ("tree", 4), ("tree", 64)])
def test_pilot_logits(name, B):
    wl = WL.make(name, n_samples=max(16, B))
    d = make_ctx(wl, max_batch=B, flags=F_NO_HOST_POOL)
    logits = torch.zeros((B, wl.pilot.O), device="cuda")
    d.predict(wl.samples[:B].copy(), hist_for(wl, B), B, logits, stream=_stream())
    r = oracle_step(wl, range(B), PL.initial_state(len(wl.tensors)), (), plan=False)
    y = logits.cpu().numpy()
    n1 = 0
    for b in range(B):
        g1, g2, o = logit_gates(y[b], r["feats"][b], wl.pilot, wl.nn_type)
        assert g2.all(), f"fp32 error bound violated at {np.where(~g2)[0][:5]}"
        n1 += int((~g1).sum())
    assert n1 == 0, f"{n1} logits outside 1e-5 relative (floored)"
    # which kernel ran: K1 (fp64 accumulation: cluster GEMV at batch 1, DMMA tiles for batches)
    assert d.query("pilot_kernel") == 0
    d.close()


@pytest.mark.parametrize("name,B", [("moe", 1), ("tiny", 1), ("moe", 8)])
def test_pilot_back_to_back_chained_history(name, B):
    """Consecutive predictions on one stream with no host sync between them (the pilot launches
    with programmatic dependent launch: its prologue overlaps the previous kernel): every
    prediction's logits match the oracle fed the previous prediction's block table (R3 history),
    and the last decode is exact."""
    wl = WL.make(name, n_samples=8 * B)
    d = make_ctx(wl, max_batch=B, flags=F_NO_HOST_POOL)
    outs = [torch.zeros((B, wl.pilot.O), device="cuda") for _ in range(8)]
    for k in range(8):
        d.predict(wl.samples[k * B:(k + 1) * B].copy(), hist_for(wl, B), B, outs[k], stream=_stream())
    torch.cuda.synchronize()
    table = ()
    r = None
    for k in range(8):
        r = oracle_step(wl, range(k * B, (k + 1) * B), PL.initial_state(len(wl.tensors)), table, plan=False)
        y = outs[k].cpu().numpy()
        for b in range(B):
            g1, g2, _ = logit_gates(y[b], r["feats"][b], wl.pilot, wl.nn_type)
            assert g1.all() and g2.all(), f"prediction {k} sample {b}"
        table = r["table"]
    for b in range(B):
        _check_prediction(d, wl, b, r["preds"][b])
    d.close()


@pytest.mark.parametrize("width", [32, 64, 128, 256, 1024, 2048])
@pytest.mark.parametrize("B", [1, 64])
def test_pilot_logits_width_sweep(width, B):
    """The width-sweep pilots ("H<w>": P512's topology at hidden width w) meet the same
    north_star gate at batch 1 and 64 (each width picks its own cluster size / samples per cluster)."""
    wl = WL.make_moe(n_samples=max(16, B), pilot_kind=f"H{width}")
    d = make_ctx(wl, max_batch=B, flags=F_NO_HOST_POOL)
    logits = torch.zeros((B, wl.pilot.O), device="cuda")
    d.predict(wl.samples[:B].copy(), hist_for(wl, B), B, logits, stream=_stream())
    torch.cuda.synchronize()
    ids = range(0, B, 7) if B > 8 else range(B)
    r = oracle_step(wl, ids, PL.initial_state(len(wl.tensors)), (), plan=False)
    y = logits.cpu().numpy()
    for i, b in enumerate(ids):
        g1, g2, _ = logit_gates(y[b], r["feats"][i], wl.pilot, wl.nn_type)
        assert g2.all() and g1.all(), f"width {width} sample {b}"
    d.close()


@pytest.mark.parametrize("name,B", [("tiny", 1), ("moe", 2), ("af", 1), ("lstm", 4)])
def test_predict_from_encoded_features(name, B):
    """The unfused entry: dyo_encode_features -> device features -> dyo_pilot_predict(feat=...)
    gives the oracle's logits (north_star gate) and decode, like the fused path."""
    wl = WL.make(name, n_samples=16)
    d = make_ctx(wl, max_batch=B, flags=F_NO_HOST_POOL)
    feat = torch.zeros((B, wl.pilot.F), device="cuda")
    logits = torch.zeros((B, wl.pilot.O), device="cuda")
    d.encode(wl.samples[:B].copy(), hist_for(wl, B), B, feat, _stream())
    d.predict(wl.samples[:B].copy(), hist_for(wl, B), B, logits, feat=feat, stream=_stream())
    r = oracle_step(wl, range(B), PL.initial_state(len(wl.tensors)), (), plan=False)
    assert np.array_equal(feat.cpu().numpy().astype(np.float64), np.stack(r["feats"]))
    y = logits.cpu().numpy()
    for b in range(B):
        g1, g2, _ = logit_gates(y[b], r["feats"][b], wl.pilot, wl.nn_type)
        assert g1.all() and g2.all()
        _check_prediction(d, wl, b, r["preds"][b])
    d.close()


def _check_prediction(d, wl, b, pred):
    K, blocks, choices, rows = d.prediction(b, wl.K_max, len(A.sites(wl.program)), _stream())
    if A.nested_ids(wl.program):          # R16: nested executions resolved by the host traversal
        assert d.nested(b) == pred.nested
        assert d.matched(b) == int(pred.matched)
    assert K == len(pred.groups)
    assert [tuple(r) for r in rows.tolist()] == pred.groups
    assert [tuple(v) for v in blocks.tolist()] == [tuple(v) for v in pred.blocks]
    assert choices.tolist() == pred.choices
    for g in range(K):
        ent = d.group_entries(b, g, stream=_stream())
        assert [tuple(e) for e in ent.tolist()] == [(t, m, int(f)) for t, m, f in pred.W[g]], f"group {g}"


@pytest.mark.parametrize("name,B", [("tiny", 1), ("tiny", 8), ("moe", 1), ("moe", 4), ("af", 2), ("lstm", 8),
                                    ("tree", 1), ("tree", 8), ("tree", 64)])
def test_decode(name, B):
    wl = WL.make(name, n_samples=max(16, B))
    d = make_ctx(wl, max_batch=B, flags=F_NO_HOST_POOL)
    d.predict(wl.samples[:B].copy(), hist_for(wl, B), B, stream=_stream())
    r = oracle_step(wl, range(B), PL.initial_state(len(wl.tensors)), (), plan=False)
    for b in range(B):
        assert not r["preds"][b].near_ties
        _check_prediction(d, wl, b, r["preds"][b])
    d.close()


def _run_plan_steps(wl, steps, B=1, policy=None, flags=F_NO_HOST_POOL):
    d = make_ctx(wl, max_batch=B, flags=flags, policy=policy)
    st = PL.initial_state(len(wl.tensors))
    table = ()
    for s in range(steps):
        ids = [(s * B + i) % len(wl.samples) for i in range(B)]
        r = oracle_step(wl, ids, st, table, policy)
        d.predict(wl.samples[ids].copy(), hist_for(wl, B), B, stream=_stream())
        if r["err"] is not None:
            with pytest.raises(Exception) as ei:
                d.plan(stream=_stream())
            assert getattr(ei.value, "status", None) == -3
        else:
            K = d.plan(stream=_stream())
            assert K == len(r["trs"])
            for j, tr in enumerate(r["trs"]):
                info = d.plan_info(j)
                assert (info["half"], info["h2d"], info["d2h"], info["d2d"], info["need"]) == \
                    (tr.half, tr.h2d, tr.d2h, tr.d2d, tr.need), f"step {s} transition {j}"
                assert gpu_lists(d, j) == tr_lists(tr), f"step {s} transition {j}"
                # R20: SHARE'd tensors (their entry records point into half 1-m) and late_all
                assert (info["n_share"], info["late_all"]) == (len(tr.share), int(tr.late_all)), f"step {s} tr {j}"
                if tr.share:
                    ent = {int(e[0]): int(e[3]) for e in d.plan_records(j, 5)}
                    assert all(ent[t] == dst for t, dst in tr.share), f"step {s} transition {j}"
            st = r["state"]
        table = r["table"]
    return d


@pytest.mark.parametrize("policy", [0, 1, 2, 3])
@pytest.mark.parametrize("name,steps,B", [("tiny", 8, 1), ("tiny", 3, 8), ("moe", 6, 1), ("af", 3, 1)])
def test_plan_bitexact(name, steps, B, policy):
    wl = WL.make(name, n_samples=32)
    _run_plan_steps(wl, steps, B, policy).close()


@pytest.mark.parametrize("budget_mib", [160, 256, 384])
def test_plan_tight_budgets_and_errors(budget_mib):
    """Tight budgets: evictions with writeback, compaction, and DYO_E_BUDGET (transactional)."""
    wl = WL.make("tiny", n_samples=32)
    wl.budget = budget_mib << 20
    for policy in (0, 1, 3):
        _run_plan_steps(wl, 10, 1, policy).close()


def test_unplanted_pilot_random_partitions():
    wl = WL.make("tiny", n_samples=32)
    wl2 = WL.make_tiny(seed=3, n_samples=32, planted=False)
    wl2.budget = 4 << 30
    _run_plan_steps(wl2, 4, 1, 1).close()
    _ = wl


def test_state_unchanged_after_budget_error():
    wl = WL.make("tiny", n_samples=32)
    d = make_ctx(wl, max_batch=1, flags=F_NO_HOST_POOL)
    st = PL.initial_state(len(wl.tensors))
    r0 = oracle_step(wl, [0], st, ())
    d.predict(wl.samples[[0]].copy(), None, 1, stream=_stream())
    d.plan(stream=_stream())
    # a prediction whose group needs more than H: an all-zero block head -> one group = whole path
    big = WL.make_tiny(seed=0, n_samples=32, planted=False)
    big.pilot.weights["out.W"][:80] = 0
    big.pilot.weights["out.b"][:80] = 0
    d2 = make_ctx(big, max_batch=1, flags=F_NO_HOST_POOL)
    d2.predict(big.samples[[0]].copy(), None, 1, stream=_stream())
    with pytest.raises(Exception):
        d2.plan(stream=_stream())
    # after the failure the committed state is the initial one: a feasible plan matches the oracle
    d2.load_pilot(wl.pilot)
    d2.predict(wl.samples[[0]].copy(), None, 1, stream=_stream())
    K = d2.plan(stream=_stream())
    assert K == len(r0["trs"]) and gpu_lists(d2, 0) == tr_lists(r0["trs"][0])
    d.close(); d2.close()


@pytest.mark.parametrize("name,steps", [("tiny", 4), ("moe", 3)])
def test_plan_bitexact_global_state_path(name, steps, monkeypatch):
    """The planner's global-memory state path (used when the per-tensor state does not fit in
    shared memory) must give the same plans as the shared-memory path."""
    monkeypatch.setenv("DYO_PLAN_GLOBAL_STATE", "1")
    wl = WL.make(name, n_samples=32)
    _run_plan_steps(wl, steps, 1, 1).close()


def _planted_path_tiny(choices, seed=0):
    """tiny without a branch head whose block head is planted with the exact block vectors of
    one path cut in 8 even groups (oracle values; R4 scaling is exact in fp32)."""
    wl = WL.make_tiny(seed=seed, n_samples=32, branch_head=False)
    from oracle import decode as D
    rows = A.resolve(wl.program, choices)
    L = len(rows)
    cuts = [(k * L // 8, (k + 1) * L // 8) for k in range(8)]
    Wo, bo = wl.pilot.weights["out.W"], wl.pilot.weights["out.b"]
    Wo[:80] = 0
    bo[:80] = 0
    for k, (s, e) in enumerate(cuts):
        v = A.block10(rows[s:e])
        for i in range(10):
            bo[10 * k + i] = np.float32(v[i] / (16.0 if i < 7 else 1024.0))
    return wl


@pytest.mark.parametrize("B", [1, 4])
@pytest.mark.parametrize("planted", [None, [1, 0, 2], [0, 1, 1]])
def test_decode_traversal(B, planted):
    """No branch head: the paper's traversal on the host inside dyo_pilot_predict,
    then the device decode of the chosen path; exact-match and fallback cases."""
    wl = WL.make_tiny(n_samples=32, branch_head=False) if planted is None else _planted_path_tiny(planted)
    d = make_ctx(wl, max_batch=B, flags=F_NO_HOST_POOL)
    d.predict(wl.samples[:B].copy(), None, B, stream=_stream())
    r = oracle_step(wl, range(B), PL.initial_state(len(wl.tensors)), ())
    for b in range(B):
        p = r["preds"][b]
        assert not p.near_ties
        assert d.matched(b) == int(p.matched)
        if planted is not None:
            assert p.matched
        _check_prediction(d, wl, b, p)
    d.close()


def test_plan_bitexact_traversal():
    wl = _planted_path_tiny([1, 1, 0])
    _run_plan_steps(wl, 4, 2, 1).close()


@pytest.mark.parametrize("policy", [0, 1, 3])
def test_plan_bitexact_lstm_scaled(policy):
    """Var-length LSTM (configs[3] variant): per-timestep / per-sample tensors (R13), reversed
    backward loop, batch of 8 predictions planned as one sequence, two consecutive steps."""
    wl = WL.make_lstm(n_samples=32, batch=8, max_len=96)
    _run_plan_steps(wl, 2, 8, policy).close()


def test_plan_bitexact_lstm_fullsize():
    wl = WL.make_lstm(n_samples=16)
    _run_plan_steps(wl, 1, 8, 1).close()


@pytest.mark.parametrize("policy", [1, 3])
def test_plan_bitexact_lstm_batch64_bench_config(policy):
    """The bench's LSTM configuration: 64 predictions (K1-TC + batch decode), 1,024 transitions
    planned as one sequence, RETAIN (+ SHARE, R20); every record of every transition bit-exact,
    one host sync."""
    wl = WL.make("lstm", n_samples=64)
    d = _run_plan_steps(wl, 1, 64, policy)
    assert d.query("plan_syncs") == 1
    assert d.query("pilot_kernel") == 0
    d.close()


@pytest.mark.parametrize("policy", [0, 1, 3])
def test_plan_bitexact_tree_scaled(policy):
    """Tree-LSTM (configs[3] primary): nested leaf/internal site per node (R16), per-(sample,
    node) tensors (R13), batch of 8 predictions planned as one sequence, two steps."""
    wl = WL.make("tree", n_samples=32, batch=8, max_leaves=24, budget=64 << 20)
    _run_plan_steps(wl, 2, 8, policy).close()


def test_plan_bitexact_tree_batch64_bench_config():
    """The bench's Tree-LSTM configuration: 64 predictions, 1,024 transitions, RETAIN."""
    wl = WL.make("tree", n_samples=64)
    d = _run_plan_steps(wl, 1, 64, 1)
    assert d.query("plan_syncs") == 1
    d.close()


def test_decode_tree_random_pilot_fallback():
    """An unplanted (random) Tree-LSTM pilot: the nested executions fall back to the closest
    operator count, exactly as the oracle."""
    wl = WL.make("tree", n_samples=16, batch=4)
    rng = np.random.default_rng(5)
    Wo = wl.pilot.weights["out.W"]
    Wo[:10 * wl.K_max] = rng.uniform(-1, 1, size=Wo[:10 * wl.K_max].shape).astype(np.float32)
    wl.pilot.weights["out.b"][:10 * wl.K_max] = np.float32(2.0)
    d = make_ctx(wl, max_batch=4, flags=F_NO_HOST_POOL)
    d.predict(wl.samples[:4].copy(), hist_for(wl, 4), 4, stream=_stream())
    r = oracle_step(wl, range(4), PL.initial_state(len(wl.tensors)), (), plan=False)
    for b in range(4):
        assert not r["preds"][b].near_ties
        _check_prediction(d, wl, b, r["preds"][b])
    d.close()


def test_residency_matches_oracle_state():
    """dyo_residency: after each plan, every tensor's device address is the arena base +
    half x H + offset of the oracle's state, NULL for tensors on the host."""
    wl = WL.make("moe", n_samples=8)
    d = make_ctx(wl, max_batch=1, flags=F_NO_HOST_POOL)
    base, H = d.arena()
    st = PL.initial_state(len(wl.tensors))
    table = ()
    for s in range(3):
        r = oracle_step(wl, [s], st, table)
        d.predict(wl.samples[[s]].copy(), hist_for(wl, 1), 1, stream=_stream())
        d.plan(stream=_stream())
        st, table = r["state"], r["table"]
        for t in range(len(wl.tensors)):
            want = None if st.loc[t] == PL.HOST else base + st.loc[t] * H + st.off[t]
            assert d.residency(t) == want, f"step {s} tensor {t}"
    d.close()


@pytest.mark.parametrize("name,B", [("moe", 64), ("af", 64), ("lstm", 64), ("moe", 20), ("moe", 100)])
def test_pilot_logits_tensor_cores(name, B):
    """Opt-in K1-TC (DYO_F_PILOT_TC: tcgen05 kind::tf32, 3xTF32 split) for batches >= 16.
    fp32-accumulating tensor cores: every logit within 1e-5 of its magnitude scale
    max(|o|, sum |w z| + |b|) (reading R14) and within the rigorous fp32 error bound; gate-1
    misses are counted and must be cancellation: |o| below a quarter of the logit's scale, i.e. a
    condition number above 4, where fp32 accumulation (~2.4e-6 x scale measured) cannot reach
    1e-5 x |o|; decisions identical to the oracle's. The default batch path (fp64 DMMA) meets
    gate 1 outright (test_pilot_logits)."""
    wl = WL.make(name, n_samples=max(16, B))
    d = make_ctx(wl, max_batch=B, flags=F_NO_HOST_POOL | F_PILOT_TC)
    logits = torch.zeros((B, wl.pilot.O), device="cuda")
    d.predict(wl.samples[:B].copy(), hist_for(wl, B), B, logits, stream=_stream())
    assert d.query("pilot_kernel") == 1, "the tensor-core kernel did not run"
    r = oracle_step(wl, range(B), PL.initial_state(len(wl.tensors)), (), plan=False)
    y = logits.cpu().numpy()
    n1, worst, worst_s, n_cancel, worst_rel = 0, 0.0, 0.0, 0, 0.0
    for b in range(B):
        g1, g2, o, scale = logit_gates(y[b], r["feats"][b], wl.pilot, wl.nn_type, with_scale=True)
        err = np.abs(y[b].astype(np.float64) - o)
        assert g2.all(), f"sample {b}: fp32 error bound violated at {np.where(~g2)[0][:5]}"
        den_s = np.maximum(np.abs(o), scale)
        rel_s = np.divide(err, den_s, out=np.where(err > 0, np.inf, 0.0), where=den_s > 0)
        worst_s = max(worst_s, float(rel_s.max()))
        wide = np.abs(o) >= 0.1 * scale
        if wide.any():
            worst_rel = max(worst_rel, float((err[wide] / np.abs(o[wide])).max()))
        miss = ~g1
        n1 += int(miss.sum())
        n_cancel += int((miss & (np.abs(o) < 0.25 * scale)).sum())
        den = np.maximum(np.abs(o), 1e-3 * np.abs(o).max())
        worst = max(worst, float((err / den).max()))
    print(f"{name} B={B}: worst err/scale {worst_s:.3e}; worst err/|o| where |o| >= scale/10 {worst_rel:.3e}; "
          f"gate-1 misses {n1} (cancellation {n_cancel}), worst floored relative {worst:.3e}")
    assert worst_s <= 1e-5, "componentwise relative error above 1e-5 (R14)"
    # survey C3: a gate-1 miss that passes gate 2 must be cancellation (|o| << its scale)
    assert n1 == n_cancel, f"{n1 - n_cancel} gate-1 misses are not cancellation"
    # decisions: identical, except a branch-head argmax whose top-2 gap in the oracle's logits is
    # inside the path's error (2 x 1e-5 x the site's largest magnitude scale): a documented tie
    from oracle import afm as AF
    sites = AF.sites(wl.program)
    n_tie = 0
    for b in range(B):
        p = r["preds"][b]
        K, blocks, choices, rows = d.prediction(b, wl.K_max, len(sites), _stream())
        if choices.tolist() != p.choices:
            _, _, o, scale = logit_gates(y[b], r["feats"][b], wl.pilot, wl.nn_type, with_scale=True)
            off = 10 * wl.K_max
            for i, st_ in enumerate(sites):
                if st_.tie >= 0:
                    continue
                nch = AF.n_choices(st_)
                if choices[i] != p.choices[i]:
                    lg = o[off:off + nch]
                    gap = abs(lg[choices[i]] - lg[p.choices[i]])
                    assert gap <= 2e-5 * scale[off:off + nch].max(), f"sample {b} site {i}: not a near-tie"
                off += nch
            n_tie += 1
            continue
        _check_prediction(d, wl, b, p)
    print(f"{name} B={B}: {n_tie} predictions with a documented argmax near-tie")
    assert n_tie == 0, "decisions differ from the oracle's on a seeded config"
    d.close()


def test_plan_async_wait_overlaps_migration_and_guards():
    """dyo_plan_async / dyo_plan_wait: the same plan as dyo_plan (records bit-exact with the
    oracle), the previous plan's transitions may be enqueued in between, and the calls that would
    race with the running planner are refused (DYO_E_STATE = -5)."""
    wl = WL.make("moe", n_samples=16)
    d = make_ctx(wl, max_batch=1)
    st = PL.initial_state(len(wl.tensors))
    table = ()
    cs = _stream()
    prev_K = 0
    for s in range(3):
        r = oracle_step(wl, [s], st, table)
        d.predict(wl.samples[[s]].copy(), hist_for(wl, 1), 1, stream=cs)
        d.plan_async(stream=cs)
        with pytest.raises(Exception) as ei:
            d.predict(wl.samples[[s]].copy(), hist_for(wl, 1), 1, stream=cs)
        assert getattr(ei.value, "status", None) == -5
        with pytest.raises(Exception) as ei:
            d.plan_async(stream=cs)
        assert getattr(ei.value, "status", None) == -5
        for j in range(prev_K):                     # the previous plan migrates meanwhile
            d.migrate(j, cs)
        K = d.plan_wait()
        assert K == len(r["trs"])
        for j, tr in enumerate(r["trs"]):
            assert gpu_lists(d, j) == tr_lists(tr), f"step {s} transition {j}"
        with pytest.raises(Exception) as ei:
            d.plan_wait()
        assert getattr(ei.value, "status", None) == -5
        prev_K = K
        st, table = r["state"], r["table"]
    for j in range(prev_K):
        d.migrate(j, cs)
    torch.cuda.synchronize()
    d.close()
