"""§8(f) rows 2 and 4 measured on the GPU (one JSON line):
  partition: Sentinel-style overlap partition (R18) of full MoE traces vs the L275 heuristics
             (exposed migration time, the E13 shape) at two budgets; GPU time per label; the
             oracle's time for one label of a shorter trace (context);
  training:  dyo_trainer SGD (R19) throughput on the MoE P512 pilot (batch 64) and a fit on the
             tiny workload's overlap labels: decoded-choice accuracy of the T32 pilot before / after;
  width:     pilot latency vs hidden width H = 32 .. 2048, batch 1 and 64.
usage: python tools/bench_labels.py [--quick]"""
import json, os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch
import workloads as WL
from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo, Trainer

quick = "--quick" in sys.argv
dev = torch.device("cuda", 0)
s0 = torch.cuda.current_stream()
out = {}


def op_list(wl):
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


# ---- partition (R18) -----------------------------------------------------------------------
wl = WL.make("moe", n_samples=32)
d = Dyo(wl.budget, wl.align, wl.policy, max_batch=1, flags=4)
d.load(wl)
op_ns = [WL.op_time_ns(o) for o in op_list(wl)]
res = {}
for budget_gib in (3.0, 0.5, 0.25):
    H = int(budget_gib * (1 << 30)) // 2
    agg = {m: [] for m in ("overlap", "even_ops", "even_time", "even_size")}
    feas = {m: 0 for m in agg}
    t_label = []
    n = 8 if quick else 32
    for s in range(n):
        ch = [max(c, 0) for c in WL.actual_choices(wl, s)]
        ops, its = d.trace_path(ch)
        for m in agg:
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            cuts, ex, ok = d.partition(ops, its, 0, op_ns, wl.K_max, m, H, 50_000)
            if m == "overlap":
                t_label.append(time.perf_counter() - t0)
            if ok:
                agg[m].append(ex)
                feas[m] += 1
    L = len(ops)
    res[f"B={budget_gib}GiB"] = {
        "trace_rows": L, "K": wl.K_max, "samples": n, "bw_GBps": 50,
        "mean_exposed_us": {m: (round(float(np.mean(v)) / 1e3, 2) if v else None) for m, v in agg.items()},
        "feasible": feas,
        "overlap_vs_best_heuristic": (round(1.0 - np.mean(agg["overlap"]) / min(np.mean(v) for k, v in agg.items()
                                                                               if k != "overlap" and v), 4)
                                      if agg["overlap"] and any(v for k, v in agg.items() if k != "overlap") else None),
        "gpu_ms_per_label": round(1e3 * float(np.median(t_label)), 3)}
d.close()
out["partition"] = res

# the same comparison on the AlphaFold-shaped trace over a budget sweep (E13 on the E7 sweep,
# P:L249-L253, L275): recycle-1 samples (path <= 4096 rows), K = 32 blocks
wl = WL.make("af", n_samples=64)
d = Dyo(wl.budget, wl.align, wl.policy, max_batch=1, flags=4)
d.load(wl)
op_ns = [WL.op_time_ns(o) for o in op_list(wl)]
paths = []
for s in range(64):
    ch = [max(c, 0) for c in WL.actual_choices(wl, s)]
    ops, its = d.trace_path(ch)
    if len(ops) <= 4096:
        paths.append((ops, its))
    if len(paths) >= (4 if quick else 8):
        break
res = {}
Kaf = 32
for budget_gib in (1.0, 2.0, 4.0, 8.0):
    H = int(budget_gib * (1 << 30)) // 2
    agg = {m: [] for m in ("overlap", "even_ops", "even_time", "even_size")}
    feas = {m: 0 for m in agg}
    for ops, its in paths:
        for m in agg:
            cuts, ex, ok = d.partition(ops, its, 0, op_ns, Kaf, m, H, 50_000)
            if ok:
                agg[m].append(ex)
                feas[m] += 1
    res[f"B={budget_gib}GiB"] = {
        "trace_rows": [len(p[0]) for p in paths], "K": Kaf, "samples": len(paths), "bw_GBps": 50,
        "mean_exposed_us": {m: (round(float(np.mean(v)) / 1e3, 2) if v else None) for m, v in agg.items()},
        "feasible": feas}
d.close()
out["partition_af_sweep"] = res

# ---- training (R19) ------------------------------------------------------------------------
wl = WL.make("moe", n_samples=64)
B = 64
feat = torch.zeros((B, wl.pilot.F), device=dev)
dd = Dyo(wl.budget, wl.align, wl.policy, max_batch=B, flags=4)
dd.load(wl)
dd.encode(wl.samples[:B].copy(), np.tile(wl.hist_ids.astype(np.int32), (B, 1)), B, feat, s0.cuda_stream)
tgt = torch.rand((B, wl.pilot.O), device=dev)
tr = Trainer(wl.pilot, wl.nn_type, B)
for _ in range(3):
    tr.step(feat, tgt, B, lr=1e-5, stream=s0.cuda_stream, want_loss=False)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
n_steps = 20 if quick else 100
e0.record(s0)
for _ in range(n_steps):
    tr.step(feat, tgt, B, lr=1e-5, stream=s0.cuda_stream, want_loss=False)
e1.record(s0)
e1.synchronize()
ms = e0.elapsed_time(e1) / n_steps
tr.close()
dd.close()
out["training_moe_p512"] = {"batch": B, "ms_per_step": round(ms, 3), "samples_per_s": round(B / (ms * 1e-3), 1),
                            "lr": 1e-5, "note": "fp64 SGD kernels (R19), P512 pilot, O = 544"}

# tiny: fit the T32 pilot to overlap labels (K = 8) and the actual choices; decoded-choice accuracy
wl = WL.make("tiny", n_samples=256)
d = Dyo(wl.budget, wl.align, wl.policy, max_batch=64, flags=4)
d.load(wl)
op_ns = [WL.op_time_ns(o) for o in op_list(wl)]
H = wl.budget // 2
n_train = 192
targets = np.zeros((256, wl.pilot.O), np.float32)
acts = []
from_sites = None
for s in range(256):
    ch = [max(c, 0) for c in WL.actual_choices(wl, s)]
    acts.append(ch)
    ops, its = d.trace_path(ch)
    cuts, ex, ok = d.partition(ops, its, 0, op_ns, wl.K_max, "overlap", H, 50_000)
    # label block vectors from the library's own decode of the rows: counts + signature sums
    # come from the trace itself (block10 of each block) - computed here from the op table
    sig = []
    ol = op_list(wl)
    for j in range(len(cuts) - 1):
        v = [cuts[j + 1] - cuts[j]] + [0] * 9
        for r in range(cuts[j], cuts[j + 1]):
            o = ops[r]
            if o >= 0:
                op = ol[o]
                dims = [sum(sh[k] for sh in op.inputs if len(sh) > k) for k in range(3)]
                for e, x in enumerate(list(op.idioms) + dims):
                    v[1 + e] += x
        sig.append(v)
    for k, v in enumerate(sig):
        for e in range(10):
            targets[s, 10 * k + e] = v[e] / (16.0 if e < 7 else 1024.0)
    off = 10 * wl.K_max
    # branch head: one-hot of each free site's actual choice (site order of the arch)
    import itertools
    ns = 0
    def walk(items):
        for it in items:
            if isinstance(it, (WL.If, WL.Loop)):
                yield it
                if isinstance(it, WL.If):
                    for br in it.branches:
                        yield from walk(br)
                else:
                    yield from walk(it.body)
    for i, site in enumerate(walk(wl.program)):
        if site.tie >= 0:
            continue
        nch = len(site.branches) if isinstance(site, WL.If) else site.hi - site.lo + 1
        targets[s, off + ch[i]] = 1.0
        off += nch
feats = torch.zeros((256, wl.pilot.F), device=dev)
for b0 in range(0, 256, 64):
    d.encode(wl.samples[b0:b0 + 64].copy(), None, 64, feats[b0:b0 + 64], s0.cuda_stream)
T = torch.from_numpy(targets).to(dev)


def accuracy(spec):
    dp = Dyo(wl.budget, wl.align, wl.policy, max_batch=64, flags=4)
    dp.load_arch(wl)
    dp.load_pilot(spec)
    ok = 0
    for b0 in range(n_train, 256, 64):
        nb = min(64, 256 - b0)
        dp.predict(wl.samples[b0:b0 + nb].copy(), None, nb, stream=s0.cuda_stream)
        for b in range(nb):
            _, _, choices, _ = dp.prediction(b, wl.K_max, 4096, s0.cuda_stream)
            ok += choices[:len(acts[b0 + b])].tolist() == acts[b0 + b]
    dp.close()
    return ok / (256 - n_train)


acc0 = accuracy(wl.pilot)
tr = Trainer(wl.pilot, wl.nn_type, 64)
losses = []
epochs = 20 if quick else 200
for ep in range(epochs):
    for b0 in range(0, n_train, 64):
        L = tr.step(feats[b0:b0 + 64], T[b0:b0 + 64], 64, lr=0.01, stream=s0.cuda_stream, want_loss=(b0 == 0))
        if b0 == 0:
            losses.append(L)           # the epoch's first minibatch loss (the others are not read back)
w = tr.weights()
tr.close()
import copy
spec2 = copy.deepcopy(wl.pilot)
for k, v in w.items():
    spec2.weights[k] = v.astype(np.float32)
acc1 = accuracy(spec2)
d.close()
out["training_tiny_t32"] = {"train_samples": n_train, "held_out": 256 - n_train, "epochs": epochs, "lr": 0.01,
                            "loss_first": float("%.6g" % losses[0]), "loss_last": float("%.6g" % losses[-1]),
                            "held_out_choice_accuracy_before": round(acc0, 4), "held_out_choice_accuracy_after": round(acc1, 4),
                            "labels": "overlap partition (R18, K=8) block vectors + actual choices (workloads.actual_choices)"}

# ---- width sweep ------------------------------------------------------------------
sweep = {}
for wdt in ([32, 512, 2048] if quick else [32, 64, 128, 256, 512, 1024, 2048]):
    wl = WL.make_moe(n_samples=64, pilot_kind=f"H{wdt}") if wdt != 512 else WL.make("moe", n_samples=64)
    r = {}
    for Bq in (1, 64):
        dp = Dyo(wl.budget, wl.align, wl.policy, max_batch=Bq, flags=4 | 8)
        dp.load(wl)
        desc = torch.from_numpy(wl.samples[:Bq].copy()).to(dev)
        hist = torch.from_numpy(np.tile(wl.hist_ids.astype(np.int32), (Bq, 1))).to(dev)
        for _ in range(5):
            dp.predict(desc, hist, Bq, stream=s0.cuda_stream)
        torch.cuda.synchronize()
        dp.timings(reset=True)
        nrep = 50
        for _ in range(nrep):
            dp.predict(desc, hist, Bq, stream=s0.cuda_stream)
        torch.cuda.synchronize()
        t = dp.timings(reset=True)
        r[f"b{Bq}_pilot_us"] = round(t["pilot"]["ms"] * 1e3 / t["pilot"]["launches"], 2)
        dp.close()
    sweep[wdt] = r
out["width_sweep_moe"] = sweep
print(json.dumps(out))
