"""GPU-side test harness: run the hot path through libdyo's C ABI and the oracle side by side.

Inputs for both sides come from workloads/ only; expected values come from oracle/ only."""
import numpy as np

import workloads as WL
from oracle import encode as E, pilot as P, decode as D, plan as PL, afm as A

F_NO_ZEROCOPY, F_NO_PACK, F_NO_HOST_POOL = 1, 2, 4
F_PILOT_TC = 32


def make_ctx(wl, max_batch=1, flags=0, policy=None, **kw):
    from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo
    d = Dyo(wl.budget, wl.align, wl.policy if policy is None else policy, max_batch=max_batch, flags=flags, **kw)
    d.load(wl)
    return d


def oracle_step(wl, sample_ids, state, table, policy=None, plan=True, drop=None):
    """Oracle for a batch of samples planned together (sample order); plan=False stops after
    the decode. drop = (p, seed): the planned tensor sets lose their read-first entries chosen by
    workloads.drop_prefetch (the DYO_FAULT injection); r["Ws"] holds the planned sets."""
    preds, feats, logits = [], [], []
    for b, s in enumerate(sample_ids):
        x = E.encode(wl, wl.samples[s], wl.hist_ids, table)
        y = P.forward(wl.pilot, x, wl.nn_type)
        feats.append(x)
        logits.append(y)
        preds.append(D.decode(wl, y, branch_head=wl.notes.get("branch_head", True), b=b))
    if drop is not None:
        Ws = [Wj for b, p in enumerate(preds) for Wj in WL.drop_prefetch(p.W, drop[0], drop[1], b)]
    else:
        Ws = [Wj for p in preds for Wj in p.W]
    new_table = [b for p in preds for b in p.blocks]
    if not plan:
        return dict(feats=feats, logits=logits, preds=preds, trs=[], state=state, table=new_table, err=None, Ws=Ws)
    try:
        trs, st = PL.plan(state, wl, Ws, policy)
        err = None
    except PL.BudgetError as e:
        trs, st, err = [], state, e
    return dict(feats=feats, logits=logits, preds=preds, trs=trs, state=st, table=new_table, err=err, Ws=Ws)


def hist_for(wl, B):
    if wl.h == 0:
        return None
    return np.tile(wl.hist_ids.astype(np.int32), (B, 1))


def tr_lists(tr):
    return {"evict": [list(map(int, r)) for r in tr.evict], "move": [list(r) for r in tr.move],
            "carry": [list(map(int, r)) for r in tr.carry], "alloc": [list(r) for r in tr.alloc],
            "fetch": [list(r) for r in tr.fetch]}


def gpu_lists(d, j):
    return {k: d.plan_records(j, k).tolist() for k in ("evict", "move", "carry", "alloc", "fetch")}


def logit_gates(y_gpu, x, spec, nn_type, with_scale=False):
    """Gate 1 (north_star): |g-o| <= 1e-5 * max(|o|, 1e-3 max|o|). Gate 2: rigorous fp32
    forward-error bound propagated layer by layer (gamma_n = n u / (1 - n u), u = 2^-24).
    with_scale: also return the output layer's magnitude scale sum_k |w_ik z_k| + |b_i| (the
    denominator of the tensor-core path's componentwise gate, reading R14)."""
    u = 2.0 ** -24
    w = spec.weights

    def layer(Wt, b, z, e, act):
        Wt = Wt.astype(np.float64); b = b.astype(np.float64)
        n = Wt.shape[1] + 1
        g = n * u / (1 - n * u)
        v = Wt @ z + b
        ev = np.abs(Wt) @ e + g * (np.abs(Wt) @ np.abs(z) + np.abs(b))
        if act:
            v2 = np.where(v > 0, v, 0.01 * v)
            ev = ev + u * np.abs(v2) + 1e-300
            return v2, ev
        return v, ev
    if spec.feature:
        zs, es = [], []
        for i, (off, ln, _) in enumerate(spec.feature):
            z, e = layer(w[f"feat{i}.W"], w[f"feat{i}.b"], x[off:off + ln], np.zeros(ln), True)
            zs.append(z); es.append(e)
        z, e = np.concatenate(zs), np.concatenate(es)
    else:
        z, e = x, np.zeros_like(x)
    for l in range(len(spec.mlp)):
        z, e = layer(w[f"mlp{nn_type}.{l}.W"], w[f"mlp{nn_type}.{l}.b"], z, e, True)
    scale = np.abs(w["out.W"].astype(np.float64)) @ np.abs(z) + np.abs(w["out.b"].astype(np.float64))
    o, e = layer(w["out.W"], w["out.b"], z, e, False)
    err = np.abs(y_gpu.astype(np.float64) - o)
    if with_scale:
        return err <= 1e-5 * np.maximum(np.abs(o), 1e-3 * np.abs(o).max()), err <= e * 1.01 + 1e-30, o, scale
    g1 = err <= 1e-5 * np.maximum(np.abs(o), 1e-3 * np.abs(o).max())
    g2 = err <= e * 1.01 + 1e-30
    return g1, g2, o
