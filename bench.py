#!/usr/bin/env python
"""Benchmark of the DyNN-Offload hot path (pilot -> decode -> plan -> migrate) on B200.

One *step* = one training sample of the workload: dyo_pilot_predict (fused encode + pilot MLP +
decode) -> dyo_plan (planner kernel + the one host sync) -> dyo_migrate(j) for every predicted
transition (DMA + copy kernels on a side copy stream). The headline metric (BASELINE.json) is
"pilot us/prediction; plan us; migration H2D/D2H GB/s vs PCIe Gen5 x16 peak"; `value` is the
whole-job migration throughput (algorithmic H2D + D2H bytes / step time, all ranks), and the
pilot / plan / per-direction numbers ride along in the same line.

  python bench.py [--gpus N --steps K --warmup W --config moe|tiny|af --policy 0|1]
  python bench.py --impl reference ...   (the CPU oracle, timed on the host cores)

Workload: BASELINE configs[1] (switch-MoE, 16 experts, 8x oversubscribed expert pool) unless
--config says otherwise. Inputs are synthetic (workloads/, seeded); every step moves >= 1 GiB
through HBM and PCIe, far above the 126 MB L2 ("inputs larger than L2").
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

PCIE_GEN5_X16 = 63.0          # GB/s per direction, 32 GT/s x 16 x 128/130 / 8 (theoretical)
DYO_F_TIMING = 8


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="dyo", choices=["dyo", "reference"])
    ap.add_argument("--config", default="moe", choices=["moe", "tiny", "af", "lstm", "tree"])
    ap.add_argument("--policy", type=int, default=1)
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--budget-gib", type=float, default=0.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-faults", action="store_true", help="skip the on-demand fetch measurement")
    ap.add_argument("--sm-copy", action="store_true",
                    help="DYO_F_SM_COPY: device moves by the SM vector-copy kernel (host-built work items) instead of TMA")
    ap.add_argument("--strict-order", action="store_true",
                    help="DYO_F_STRICT_ORDER: R12's whole-phase EVICT -> FETCH order instead of R21's per-range order")
    ap.add_argument("--dist-backend", default=None, help="nccl (default with CUDA) or gloo")
    ap.add_argument("--compute", default="auto", choices=["auto", "none", "emulate"],
                    help="emulate the DyNN's per-group compute with spin kernels (auto: on for af)")
    return ap.parse_args()


CONFIG_DESC = {
    "moe": "switch-MoE top-1 trace, 24 layers x 16 experts (32 MiB W_in/W_out, grads written back), "
           "3 GiB budget = 8x oversubscribed expert pool, P512 pilot (BASELINE configs[1])",
    "tiny": "tiny trace: 8 groups, 64 tensors, T32 pilot, 1 GiB budget (BASELINE configs[0])",
    "af": "AlphaFold-Evoformer-shaped trace, 48 blocks x recycle 1..4, MSA 128x256, 2 GiB budget (BASELINE configs[2])",
    "lstm": "variable-length 2-layer LSTM (length U{16..512}, 4 task heads), batch of 64 predictions planned per "
            "step, 35,860 tensors of 2-4 KiB (+ 4 MiB weights), 48 MiB budget (BASELINE configs[3], var-length variant)",
    "tree": "Tree-LSTM over random binary parse trees (leaves U{8..64}, 2n-1 node loop with a nested leaf/internal If "
            "resolved per node by the traversal, reading R16), batch of 64 predictions planned per step, 33,031 tensors "
            "of 2-4 KiB (+ 14 MiB weights/grads), 256 MiB budget (BASELINE configs[3], Tree-LSTM primary)",
}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except OSError:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0}, "fallback"


class Clocks:
    """nvidia-smi sampler running during the timed region."""

    def __init__(self, index=0):
        self.samples = []
        self.proc = None
        self.index = index

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active,"
                 "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                 "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            threading.Thread(target=self._read, daemon=True).start()
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.samples.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4) if len(s) > 3 + i and s[3 + i] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


def reduce_over_ranks(vals_max, vals_sum, backend):
    """Max of `vals_max` and sum of `vals_sum` over all ranks (timings: the slowest rank bounds the
    job; bytes: every rank's work counts). World size 1: identity."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return list(vals_max), list(vals_sum)
    dev = torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else torch.device("cpu")
    a = torch.tensor(list(vals_max), dtype=torch.float64, device=dev)
    b = torch.tensor(list(vals_sum), dtype=torch.float64, device=dev)
    dist.all_reduce(a, op=dist.ReduceOp.MAX)
    dist.all_reduce(b, op=dist.ReduceOp.SUM)
    return a.cpu().tolist(), b.cpu().tolist()


def make_workload(args, rank):
    import workloads as WL
    wl = WL.make(args.config, seed=args.seed + rank, n_samples=128)
    wl.policy = args.policy
    if args.budget_gib > 0:
        wl.budget = int(args.budget_gib * (1 << 30))
    return wl


# ---------------------------------------------------------------------------------------------
# CPU oracle legs (the only place bench.py executes oracle/)
# ---------------------------------------------------------------------------------------------

def oracle_steps(wl, n_steps, budget_s=None):
    """Run the oracle as it stands for n_steps samples: encode, pilot (fp64), decode, plan (pure
    Python), then the step's algorithmic bytes copied by numpy between a host buffer pair (the
    oracle's byte model moves exactly these bytes; full-size arenas do not fit its numpy model,
    so the copy runs through 256 MiB buffers). Returns (bytes, seconds, steps_done)."""
    import numpy as np
    from threadpoolctl import threadpool_limits
    from oracle import run as OR, plan as PL
    st = PL.initial_state(len(wl.tensors))
    table = ()
    buf_a = np.ones(256 << 20, np.uint8)
    buf_b = np.zeros(256 << 20, np.uint8)
    total_b, t0, done = 0, time.perf_counter(), 0
    B = wl.notes.get("batch", 1)
    bs = min(B, wl.notes.get("oracle_batch", B))     # bounded sample of a batched step
    with threadpool_limits(limits=1):
        for s in range(n_steps):
            if B == 1:
                r = OR.step(wl, s % len(wl.samples), st, table)
                st, table, trs = r.state, r.pred.blocks, r.transitions
            else:
                ids = [(s * bs + i) % len(wl.samples) for i in range(bs)]
                preds, trs, st, _ = OR.step_batch(wl, ids, st, table)
                table = [v for p in preds for v in p.blocks]
            nbytes = sum(t.h2d + t.d2h for t in trs)
            left = nbytes
            while left > 0:
                n = min(left, buf_a.size)
                np.copyto(buf_b[:n], buf_a[:n])
                left -= n
            total_b += nbytes
            done += 1
            if budget_s is not None and time.perf_counter() - t0 > budget_s:
                break
    return total_b, time.perf_counter() - t0, done


def oracle_components(wl, budget_s=6.0):
    """The oracle's per-component times on one host core (B = 1 steps): encode + pilot forward
    (us/prediction), decode (us/prediction) and plan (us/step) - the CPU counterparts of the
    GPU line's pilot_us_per_prediction and plan_us."""
    from threadpoolctl import threadpool_limits
    from oracle import encode as E, pilot as P, decode as D, plan as PL
    st = PL.initial_state(len(wl.tensors))
    table = ()
    t_pilot = t_dec = t_plan = 0.0
    n = 0
    t_start = time.perf_counter()
    with threadpool_limits(limits=1):
        while time.perf_counter() - t_start < budget_s:
            smp = wl.samples[n % len(wl.samples)]
            t0 = time.perf_counter()
            x = E.encode(wl, smp, wl.hist_ids, table)
            y = P.forward(wl.pilot, x, wl.nn_type)
            t1 = time.perf_counter()
            pred = D.decode(wl, y, branch_head=wl.notes.get("branch_head", True))
            t2 = time.perf_counter()
            try:
                _, st = PL.plan(st, wl, pred.W, None)
            except PL.BudgetError:
                st = PL.initial_state(len(wl.tensors))
            t3 = time.perf_counter()
            table = pred.blocks
            t_pilot += t1 - t0
            t_dec += t2 - t1
            t_plan += t3 - t2
            n += 1
    return {"pilot_us_per_prediction": round(t_pilot / n * 1e6, 1), "decode_us_per_prediction": round(t_dec / n * 1e6, 1),
            "plan_us_per_step": round(t_plan / n * 1e6, 1), "steps": n, "cores": 1}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    wl = make_workload(args, 0)
    oracle_steps(wl, max(args.warmup, 1))
    b, sec, n = oracle_steps(wl, args.steps)
    v = b / sec / 1e9
    out = {"metric": "migration GB/s (pilot us/prediction; plan us; H2D/D2H vs PCIe Gen5 x16)",
           "impl": "reference", "value": round(v, 4), "unit": "GB/s", "n_gpus": args.gpus, "steps": n,
           "warmup": args.warmup, "ms_per_step": round(sec / n * 1e3, 3), "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "f64 pilot / int64 plan / u8 bytes",
           "data": "synthetic", "config": {"workload": args.config, "desc": CONFIG_DESC[args.config]},
           "cpu_baseline": {"value": round(v, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                            "sample": f"{n} full oracle steps (pure Python encode/pilot/decode/plan + numpy copy of "
                                      f"the step's algorithmic bytes), 1 host core"},
           "e2e": {"value": round(v, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


# ---------------------------------------------------------------------------------------------
# B200 leg
# ---------------------------------------------------------------------------------------------

def pilot_latency(torch, wl, dev, desc_dev, hist64, nS, s0):
    """Batch-1 pilot latency three ways (survey section 8(d)): single-shot host-observed (call ->
    stream synchronised), CUDA-graph replay of 100 back-to-back predictions / 100, and the floor
    = a graph of 100 empty launches of the pilot's shape (one cluster, L cluster barriers for its
    L dependent stages) / 100."""
    import numpy as np
    from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo
    sp = wl.pilot
    wbytes = 4 * (sum((ln + 1 + 3) // 4 * 4 * o for _, ln, o in sp.feature) + sum((i + 1 + 3) // 4 * 4 * o for i, o in sp.mlp)
                  + (sp.out_in + 1 + 3) // 4 * 4 * sp.O)
    C = 1 if wbytes <= (64 << 10) else (4 if wbytes <= (512 << 10) else 16)
    L = (1 if sp.feature else 0) + len(sp.mlp) + 1
    g1 = Dyo(wl.budget, wl.align, wl.policy, max_batch=1, device=dev, flags=4)
    g1.load(wl)
    h1 = hist64[:1] if hist64 is not None else None
    out = {"cluster": C, "stages": L}
    try:
        ss = []
        for i in range(40):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            g1.predict(desc_dev[i % nS: i % nS + 1], h1, 1, stream=s0.cuda_stream)
            s0.synchronize()
            ss.append((time.perf_counter() - t0) * 1e6)
        out["single_shot_us"] = round(float(np.median(ss[5:])), 2)
        if g1.query("host_decode"):
            # the decode of this arch runs on the host (nested sites, R16): one stream sync per
            # predict, so there is no graph to replay
            out["note"] = "host-side decode (nested sites, R16): single-shot only, no graph replay"
            g1.close()
            return out
        cs = torch.cuda.Stream()
        for _ in range(3):
            g1.predict(desc_dev[:1], h1, 1, stream=cs.cuda_stream)
        torch.cuda.synchronize()

        def replay(fn):
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=cs):
                for i in range(100):
                    fn(i, torch.cuda.current_stream().cuda_stream)
            with torch.cuda.stream(cs):              # replay() launches on the current stream
                g.replay()
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(cs)
                for _ in range(10):
                    g.replay()
                e1.record(cs)
            e1.synchronize()
            return e0.elapsed_time(e1) * 1e3 / 1000
        out["graph_replay_us"] = round(replay(lambda i, st: g1.predict(desc_dev[i % nS: i % nS + 1], h1, 1, stream=st)), 2)
        out["floor_us"] = round(replay(lambda i, st: g1.debug_floor(C, L, st)), 2)
        # single-CTA empty launch: the planner's latency floor (survey 8(d) "fraction of the
        # single-launch floor")
        out["single_cta_launch_floor_us"] = round(replay(lambda i, st: g1.debug_floor(1, 0, st)), 2)
        out["floor_frac"] = round(out["floor_us"] / out["graph_replay_us"], 4)
        out["note"] = ("floor = empty launch of the pilot's cluster shape with one cluster barrier per dependent stage, "
                       "graph-replayed; graph_replay_us includes the fused decode")
    except Exception as e:     # capture unsupported on this path: report what was measured
        out["error"] = str(e)[:200]
    g1.close()
    return out


def mispredict_stream(torch, wl, dev, s0, n_distinct=16, repeats=4):
    """Mis-prediction record + exact-match memo on a sample stream with
    repeats: `repeats` passes over `n_distinct` samples (history-free features, so a repeated
    sample reproduces its pilot output), the actual control flow of every sample from
    workloads.actual_choices. Reports the mis-prediction counts without and with the memo and the
    batch-1 predict time with a populated memo (the decode's hash probe) vs without. Outside the
    timed region."""
    import numpy as np
    import workloads as WLm
    from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo
    if not wl.notes.get("branch_head", True):
        return None
    out = {"samples": n_distinct, "repeats": repeats}
    acts = [WLm.actual_choices(wl, i) for i in range(n_distinct)]
    desc = torch.from_numpy(wl.samples[:n_distinct].copy()).to(dev)
    for memo in (0, 1):
        d = Dyo(wl.budget, wl.align, wl.policy, max_batch=1, device=dev, flags=4)
        d.load(wl)
        if memo:
            d.memo_config(1024)
        for _ in range(repeats):
            for i in range(n_distinct):
                d.predict(desc[i:i + 1], None, 1, stream=s0.cuda_stream)
                d.report(0, acts[i])
        st = d.memo_stats()
        out["with_memo" if memo else "without_memo"] = {"mispredictions": st["mispredictions"], "memo_hits": st["hits"],
                                                         "live_entries": st["live"]}
        # predict time (stream back-to-back, device span) with this ctx's memo state
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s0)
        for k in range(200):
            d.predict(desc[k % n_distinct: k % n_distinct + 1], None, 1, stream=s0.cuda_stream)
        e1.record(s0)
        e1.synchronize()
        out["with_memo" if memo else "without_memo"]["pilot_us_per_prediction"] = round(e0.elapsed_time(e1) * 1e3 / 200, 2)
        d.close()
    out["note"] = ("actual control flow: workloads.actual_choices (Zipf(1.2) per site, seeded per sample); "
                   "closed form with pairwise-distinct outputs: without = repeats x m, with = m")
    return out


def fault_stream(torch, d, wl, desc_dev, hist_dev, nS, B, s0, s1, steps=4, p_drop=0.05, seed=11):
    """On-demand fetch (R17) measured with the library's fault injection: each step's read-first
    entries are dropped from the plan with probability p_drop (dyo_fault_inject), the runtime
    migrates one block ahead and asks dyo_fault_fetch for every access of the actual (undropped)
    block. Reports faults and fault bytes per step and the step time with and without drops (the
    same block-by-block protocol, wall clock, no compute emulation). Outside the timed region."""
    import numpy as np
    d.fault_config(512 << 20)
    out = {"p_drop": p_drop, "steps": steps}
    for p in (0.0, p_drop):
        d.fault_inject(p, seed)
        st0 = d.fault_stats()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for k in range(steps):
            i0 = (k * B) % nS
            d.predict(desc_dev[i0: i0 + B], hist_dev, B, stream=s0.cuda_stream)
            acts = []
            for b in range(B):
                K, _, _, _ = d.prediction(b, wl.K_max, 4096, s0.cuda_stream)   # >= n_sites (kMaxSites)
                acts += [d.group_entries(b, g, stream=s0.cuda_stream) for g in range(K)]
            Kp = d.plan(stream=s0.cuda_stream)
            for j in range(Kp):
                d.migrate(j, s1.cuda_stream)
                e = acts[j]
                modes = [int(m) for m in e[:, 1]] if len(e) else []
                d.fault_fetch(j, [int(t) for t in e[:, 0]] if len(e) else [], modes, s1.cuda_stream)
            d.fault_flush(s1.cuda_stream)
        torch.cuda.synchronize()
        ms = (time.perf_counter() - t0) * 1e3 / steps
        st1 = d.fault_stats()
        key = "with_drops" if p > 0 else "without_drops"
        out[key] = {"ms_per_step_wall": round(ms, 3),
                    "faults_per_step": round((st1["faults"] - st0["faults"]) / steps, 2),
                    "fault_bytes_per_step": int((st1["bytes"] - st0["bytes"]) / steps),
                    "slot_accesses_per_step": round((st1["resident"] - st0["resident"]) / steps, 1)}
    d.fault_inject(0.0, 0)
    d.fault_config(0)
    return out


def calibrate_spin(torch):
    """GPU cycles per microsecond of torch.cuda._sleep (the compute emulation's spin kernel)."""
    s = torch.cuda.Stream()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        torch.cuda._sleep(1000000)
        a.record(s)
        torch.cuda._sleep(20000000)
        b.record(s)
    b.synchronize()
    return 20000000 / (a.elapsed_time(b) * 1e3)


def group_compute_us(wl, j, K):
    """Emulated compute of group j (survey §8(d) M2): Evoformer-shaped blocks of ~100 GFLOP forward
    and 2x that backward at half the sustained bf16 rate (0.5 x 1398 TFLOPS) -> ~143 / ~286 us;
    the final group ~10 us. Groups past the forward recycles are backward."""
    blocks = wl.notes.get("blocks", 48)
    if j == K - 1:
        return 10.0
    return 286.0 if j >= K - 1 - blocks else 143.0


def pcie_probe(torch, nbytes=256 << 20, reps=5):
    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    res = {}
    for name, (dst, src) in (("h2d", (d, h)), ("d2h", (h, d))):
        with torch.cuda.stream(s):
            dst.copy_(src, non_blocking=True)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            for _ in range(reps):
                dst.copy_(src, non_blocking=True)
            b.record(s)
        b.synchronize()
        res[name] = nbytes * reps / (a.elapsed_time(b) * 1e-3) / 1e9
    del h, d
    return res


def run_dyo(args):
    import numpy as np
    import torch
    import torch.distributed as dist
    from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo

    # DYO_COPY_STAMPS=1 (opt-in, diagnostic): per-CTA globaltimer stamps of the record-copy kernel
    # in the instrumented pass (roofline.in_kernel); never on in the headline pass
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    # one manager per GPU; with fewer GPUs than ranks (functional tests) ranks share devices
    local = int(os.environ.get("LOCAL_RANK", "0")) % max(1, torch.cuda.device_count())
    backend = args.dist_backend or "nccl"
    if world > 1:
        dist.init_process_group(backend)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)

    wl = make_workload(args, rank)
    _log("workload built")
    B = wl.notes.get("batch", 1)          # predictions planned per step (lstm: a minibatch of 64)
    d = Dyo(wl.budget, wl.align, wl.policy, max_batch=B, device=local,
            flags=(64 if args.strict_order else 0) | (16 if args.sm_copy else 0))   # headline: uninstrumented
    d.load(wl)
    _log("ctx loaded")
    s0 = torch.cuda.current_stream()
    s1 = torch.cuda.Stream()
    desc_dev = torch.from_numpy(wl.samples.copy()).to(dev)
    hist_np = np.tile(wl.hist_ids.astype(np.int32), (B, 1)) if wl.h else None
    hist_dev = torch.from_numpy(hist_np).to(dev) if hist_np is not None else None
    nS = len(wl.samples)
    assert nS % B == 0

    # Blocks: without compute emulation, block j "starts" and "ends" when ready[j] fires, so
    # transition j's EVICT waits ready[j-2] (its half's last user) and overlaps transition j-1's
    # FETCH. With emulation, block j is a spin kernel on the compute stream after ready[j] whose
    # duration follows the workload's per-group FLOPs; migrations wait on the block-end events.
    emulate = args.compute == "emulate" or (args.compute == "auto" and args.config == "af")
    ready = [torch.cuda.Event() for _ in range(B * wl.K_max + 1)]
    bend = [torch.cuda.Event() for _ in range(B * wl.K_max + 1)]
    t_start = torch.cuda.Event()
    s_comp = torch.cuda.Stream()
    for e in ready + bend + [t_start]:
        e.record(s1)                          # materialise the cudaEvent_t handles
    cyc_per_us = calibrate_spin(torch) if emulate else 0.0
    comp_us_total = [0.0]

    per_tr = []                               # (h2d, d2h) of every transition planned (step bound)

    def plan_start(desc, hist):
        """Predict + launch the plan of one step (dyo_plan_async: the host goes on enqueuing the
        previous step's transitions while the planner runs)."""
        d.predict(desc, hist, B, stream=s0.cuda_stream)
        d.plan_async(stream=s0.cuda_stream)

    def plan_next(desc=None, hist=None):
        """Complete a plan (dyo_plan_wait: the one host sync) and read its byte counts; with
        inputs, predict + plan first."""
        if desc is not None:
            plan_start(desc, hist)
        K = d.plan_wait()
        h2d = d2h = 0
        trs = []
        for j in range(K):
            info = d.plan_info(j)
            h2d += info["h2d"]
            d2h += info["d2h"]
            if K <= 64:     # record-level detail for the R21 step bound (small plans: MoE, AF steps)
                ev = d.plan_records(j, "evict")
                fe = d.plan_records(j, "fetch")
                late = bool(info["n_carry"]) and bool(d.plan_records(j, "carry")[:, 4].any())
                trs.append((info["h2d"], info["d2h"], [(int(r[1]), int(r[3])) for r in ev if r[4]],
                            [(int(r[2]), int(r[3])) for r in fe], info["n_move"], info["late_all"], late))
            else:
                trs.append((info["h2d"], info["d2h"]))
        per_tr.append(trs)
        return K, h2d, d2h

    def enqueue(K):
        """Enqueue every transition of the oldest outstanding plan (+ the emulated compute)."""
        t_start.record(s1)
        if emulate:
            s_comp.wait_event(t_start)
        ends = bend if emulate else ready
        for j in range(K):
            half_free = ends[j - 2] if j >= 2 else t_start
            prev_done = ends[j - 1] if j >= 1 else t_start
            d.migrate(j, s1.cuda_stream, half_free.cuda_event, prev_done.cuda_event, ready[j].cuda_event)
            if emulate:
                us = group_compute_us(wl, j, K)
                comp_us_total[0] += us
                s_comp.wait_event(ready[j])
                with torch.cuda.stream(s_comp):
                    torch.cuda._sleep(int(us * cyc_per_us))
                bend[j].record(s_comp)
        if emulate:
            s1.wait_stream(s_comp)
        elif K:
            s1.wait_event(ready[K - 1])      # R21: the last ready[] may be joined off the copy stream

    def run_steps(n, first, inputs):
        """n steps with plan lookahead: step i+1 is predicted and its planner launched, step i's
        transitions are enqueued while the planner runs (dyo_plan_async), then the plan is
        completed (dyo_plan_wait) while step i migrates."""
        tot = [0, 0, 0]
        pending = plan_next(*inputs(first))
        for i in range(n):
            K, h2d, d2h = pending
            if i + 1 < n:
                plan_start(*inputs(first + i + 1))
            enqueue(K)
            tot[0] += K
            tot[1] += h2d
            tot[2] += d2h
            if i + 1 < n:
                pending = plan_next()
        return tot

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()

    _log("warmup")
    dev_inputs = lambda k: (desc_dev[(k * B) % nS: (k * B) % nS + B], hist_dev)
    run_steps(args.warmup, 0, dev_inputs)
    barrier()
    d.counters(reset=True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    tot_h2d = tot_d2h = tot_K = 0
    comp_us_total[0] = 0.0
    per_tr.clear()
    # headline pass: no timing events, no copy stamps
    with Clocks(local) as clk:
        e0.record(s0)
        tot_K, tot_h2d, tot_d2h = run_steps(args.steps, args.warmup, dev_inputs)
        s0.wait_stream(s1)
        e1.record(s0)
        e1.synchronize()
    barrier()
    comp_ms_step = comp_us_total[0] / 1e3 / args.steps if emulate else 0.0
    ms = e0.elapsed_time(e1)
    comp_only_ms = None
    if emulate:
        # the compute harness alone: the same blocks (spin kernels of the same durations, each
        # waiting an event of the copy stream, then recording its end) with no migrations, so
        # the exposure attributable to migration is the step minus this, not minus the nominal sum
        Ks = [len(t) for t in per_tr[:args.steps]]
        c0, c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        c0.record(s_comp)
        for K in Ks:
            for j in range(K):
                ready[j].record(s1)
                s_comp.wait_event(ready[j])
                with torch.cuda.stream(s_comp):
                    torch.cuda._sleep(int(group_compute_us(wl, j, K) * cyc_per_us))
                bend[j].record(s_comp)
        c1.record(s_comp)
        c1.synchronize()
        comp_only_ms = c0.elapsed_time(c1) / args.steps
    ctr = d.counters(reset=True)
    timed_trs = [t for st_ in per_tr[:args.steps] for t in st_]
    # instrumented pass (same number of steps, next samples): per-kind device times (CUDA events
    # around every launch and DMA on its stream) for the breakdown and the roofline
    _log("instrumented pass")
    d.set_timing(True)
    d.timings(reset=True)
    stamps_on = os.environ.get("DYO_COPY_STAMPS") in ("1", "2")
    if stamps_on:
        d.copy_stamps(reset=True)
    comp_save = comp_us_total[0]
    ei0, ei1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ei0.record(s0)
    run_steps(args.steps, args.warmup + args.steps, dev_inputs)
    s0.wait_stream(s1)
    ei1.record(s0)
    ei1.synchronize()
    barrier()
    ms_instr = ei0.elapsed_time(ei1)
    comp_us_total[0] = comp_save
    tm = d.timings(reset=True)
    d.set_timing(False)
    stamp_rep = None
    if stamps_on and rank == 0:
        stamp_rep = copy_stamp_report(d.copy_stamps(), os.environ.get("DYO_COPY_STAMPS_OUT"))

    _log("e2e")
    # e2e: the same steps through the public API with HOST inputs (pinned), results read back
    desc_host = torch.from_numpy(wl.samples.copy()).pin_memory()
    hist_host = torch.from_numpy(hist_np).pin_memory() if hist_np is not None else None
    barrier()
    t0 = time.perf_counter()
    host_inputs = lambda k: (desc_host[(k * B) % nS: (k * B) % nS + B].numpy(),
                             hist_host.numpy() if hist_host is not None else None)
    run_steps(args.steps, args.warmup + 2 * args.steps, host_inputs)
    s1.synchronize()
    barrier()
    e2e_s = time.perf_counter() - t0
    e2e_bytes = None

    faults = None
    if rank == 0 and not args.no_faults:
        _log("faults")
        try:
            faults = fault_stream(torch, d, wl, desc_dev, hist_dev, nS, B, s0, s1)
        except Exception as e:                  # reported, never fatal to the headline line
            faults = {"error": str(e)[:200]}
    peaks, peak_src = measured_peaks()
    _log("pilot loop")
    # pilot latency at batch 1 (the cluster GEMV kernel, decode fused) and throughput at batch 64
    # (K1-TC tensor-core kernel + two-phase decode): back-to-back predictions, device time
    dp = Dyo(wl.budget, wl.align, wl.policy, max_batch=64, device=local, flags=DYO_F_TIMING | 4)
    dp.load(wl)
    desc64 = desc_dev[:64] if nS >= 64 else desc_dev.repeat((64 + nS - 1) // nS, 1)[:64]
    hist64 = torch.from_numpy(np.tile(wl.hist_ids.astype(np.int32), (64, 1))).to(dev) if wl.h else None

    def pilot_loop(ctx, n, bsz):
        """Back-to-back predictions on one stream: a clean pass (no timing events between the
        launches, so consecutive pilots overlap by programmatic dependent launch) for the time
        per prediction, then an instrumented pass for the pilot / decode kernel split."""
        def run(k):
            for i in range(k):
                if bsz == 1:
                    ctx.predict(desc_dev[i % nS: i % nS + 1], hist64[:1] if hist64 is not None else None, 1,
                                stream=s0.cuda_stream)
                else:
                    ctx.predict(desc64, hist64, bsz, stream=s0.cuda_stream)
        ctx.set_timing(False)
        run(3)
        torch.cuda.synchronize()
        p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        p0.record(s0)
        run(n)
        p1.record(s0)
        p1.synchronize()
        ctx.set_timing(True)
        ctx.timings(reset=True)
        run(n)
        torch.cuda.synchronize()
        t = ctx.timings(reset=True)
        return (p0.elapsed_time(p1) * 1e3 / n, t["pilot"]["ms"] * 1e3 / max(1, t["pilot"]["launches"]),
                t["decode"]["ms"] * 1e3 / max(1, t["decode"]["launches"]))
    pred_us, pilot_kernel_us, decode_us = pilot_loop(dp, 200, 1)
    lat = pilot_latency(torch, wl, local, desc_dev, hist64, nS, s0)
    mis = mispredict_stream(torch, wl, local, s0) if wl.notes.get("batch", 1) == 1 else None
    b64_us, b64_kernel_us, b64_decode_us = pilot_loop(dp, 50, 64)
    b64_kern = dp.query("pilot_kernel")
    # batch work per launch: 2 x 64 x sum(in x out) over the stages (K1-TC executes x3: 3xTF32)
    sp = wl.pilot
    macs = sum(ln * o for _, ln, o in sp.feature) + sum(i * o for i, o in sp.mlp) + sp.out_in * sp.O
    tc_flop = 2.0 * 64 * macs
    dp.close()
    tc = None
    if wl.pilot.feature:
        # the opt-in tensor-core kernel K1-TC (DYO_F_PILOT_TC: tcgen05 3xTF32, reading R14) beside it
        dt = Dyo(wl.budget, wl.align, wl.policy, max_batch=64, device=local, flags=DYO_F_TIMING | 4 | 32)
        dt.load(wl)
        t_us, t_kernel_us, t_decode_us = pilot_loop(dt, 50, 64)
        assert dt.query("pilot_kernel") == 1
        dt.close()
        tf32_peak = peaks["bf16_tflops"] / 2
        tc = {"us_per_batch": round(t_us, 2), "pilot_kernel_us": round(t_kernel_us, 2),
              "decode_kernels_us": round(t_decode_us, 2), "predictions_per_s": round(64e6 / t_us, 1),
              "kernel": "pilot_tc_kernel (tcgen05 kind::tf32, 3xTF32, fp32 accumulation; reading R14 gate)",
              "tensor_roofline": {"bound": "tensor", "achieved": round(3 * tc_flop / (t_kernel_us * 1e-6) / 1e12, 4),
                                  "peak": round(tf32_peak, 1), "unit": "TFLOP/s",
                                  "frac": round(3 * tc_flop / (t_kernel_us * 1e-6) / 1e12 / tf32_peak, 6),
                                  "flop_per_launch": 3 * tc_flop,
                                  "peak_source": "TF32 dense = measured bf16 / 2 (guide's nominal ratio)"}}
    _log("probe")
    probe = pcie_probe(torch)

    # max over ranks (time), sum over ranks (work)
    (ms_max, e2e_max), (bytes_all, h2d_all, d2h_all) = reduce_over_ranks(
        [ms, e2e_s], [float(tot_h2d + tot_d2h), float(tot_h2d), float(tot_d2h)], backend)
    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        d.close()
        return

    value = bytes_all / (ms_max * 1e-3) / 1e9
    host_numa = d.query("host_numa")
    # dominant kernel of the timed region among libdyo's kernels
    kern = {k: tm[k] for k in ("pilot", "decode", "plan", "copy_d2d", "copy_zc")}
    dom = max(kern, key=lambda k: kern[k]["ms"])
    km = kern[dom]
    avg_ms = km["ms"] / max(1, km["launches"])
    if dom == "copy_d2d":
        alg = 2.0 * km["bytes"] / max(1, km["launches"])          # read + write per launch
        achieved = alg / (avg_ms * 1e-3) / 1e9
        # aggregate over the union of the launches' busy intervals: carries, compaction and packs
        # of neighbouring transitions run concurrently on three streams and share HBM, so the
        # per-launch average (above) divides one launch's bytes by a contended duration
        agg = 2.0 * km["bytes"] / (km["busy_ms"] * 1e-3) / 1e9 if km["busy_ms"] else None
        roof = {"bound": "hbm", "achieved": round(achieved, 2), "peak": peaks["hbm_gbs"], "unit": "GB/s",
                "frac": round(achieved / peaks["hbm_gbs"], 4), "traffic": None, "kernel": "copy_records_tma_kernel",
                "peak_source": peak_src, "alg_bytes_per_launch": alg, "avg_launch_us": avg_ms * 1e3,
                "aggregate_busy_gbs": round(agg, 2) if agg else None,
                "aggregate_busy_frac": round(agg / peaks["hbm_gbs"], 4) if agg else None,
                "launches_concurrent_factor": round(km["ms"] / km["busy_ms"], 3) if km["busy_ms"] else None}
        if stamp_rep and stamp_rep["launches"] == km["launches"] and stamp_rep["sum_span_us"] > 0:
            ik = 2.0 * km["bytes"] / (stamp_rep["sum_span_us"] * 1e-6) / 1e9
            roof["in_kernel"] = {"achieved": round(ik, 2), "frac": round(ik / peaks["hbm_gbs"], 4),
                                 "mean_span_us": round(stamp_rep["mean_span_us"], 2),
                                 "note": "DYO_COPY_STAMPS: globaltimer from the first CTA's entry to the last "
                                         "CTA's exit of each launch; the CUDA-event duration (achieved) also "
                                         "holds the stream's wait between the event and the kernel's start/end"}
    elif dom == "copy_zc":
        alg = km["bytes"] / max(1, km["launches"])
        achieved = alg / (avg_ms * 1e-3) / 1e9
        roof = {"bound": "pcie", "achieved": round(achieved, 2), "peak": PCIE_GEN5_X16, "unit": "GB/s",
                "frac": round(achieved / PCIE_GEN5_X16, 4), "traffic": None, "kernel": "copy_segments_kernel (zero-copy)",
                "peak_source": "theoretical PCIe Gen5 x16", "alg_bytes_per_launch": alg, "avg_launch_us": avg_ms * 1e3}
    else:
        roof = {"bound": "latency", "achieved": round(avg_ms * 1e3, 2), "peak": None, "unit": "us/launch",
                "frac": None, "traffic": None, "kernel": dom, "avg_launch_us": avg_ms * 1e3}
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            tr = json.load(f)
        t = tr.get(roof["kernel"].split()[0])
        if t and roof.get("alg_bytes_per_launch"):
            # measured DRAM bytes per algorithmic byte (one ncu capture) x this run's bytes per launch
            roof["traffic"] = round(t["dram_per_alg_byte"] * roof["alg_bytes_per_launch"])
            roof["traffic_source"] = "profiles/ncu_traffic.json: dram/alg = %s over %d launches" % (
                t["dram_per_alg_byte"], t["launches"])
    except OSError:
        pass
    shares = {k: round(v["ms"] / ms_instr, 4) for k, v in tm.items()}
    dma_h2d = tm["dma_h2d"]
    dma_d2h = tm["dma_d2h"]
    # a bound needs rates no lower than the link delivered in the step: the probe (one sample,
    # noisy on a busy box) or the DMA rate seen in the step, whichever is higher
    rate_h = max(probe["h2d"], dma_h2d["bytes"] / (dma_h2d["ms"] * 1e6) if dma_h2d["ms"] else 0.0)
    rate_d = max(probe["d2h"], dma_d2h["bytes"] / (dma_d2h["ms"] * 1e6) if dma_d2h["ms"] else 0.0)
    bound_strict_ms = step_bound_ms(timed_trs, rate_h, rate_d, strict=True) / args.steps
    # the bound of the order the run used (--strict-order: R12 everywhere)
    bound_ms = bound_strict_ms if args.strict_order else step_bound_ms(timed_trs, rate_h, rate_d) / args.steps
    bidir = max(bidir_probe(torch), bidir_probe(torch))
    bound_fluid_ms = step_bound_fluid_ms(timed_trs, rate_h, rate_d, bidir, strict=args.strict_order) / args.steps
    h2d_link = dma_h2d["bytes"] / (dma_h2d["ms"] * 1e-3) / 1e9 if dma_h2d["ms"] else None
    d2h_link = dma_d2h["bytes"] / (dma_d2h["ms"] * 1e-3) / 1e9 if dma_d2h["ms"] else None
    plan_us = tm["plan"]["ms"] * 1e3 / max(1, tm["plan"]["launches"])
    launches = (tm["pilot"]["launches"] + 3 * tm["decode"]["launches"] + tm["plan"]["launches"]
                + tm["copy_d2d"]["launches"] + tm["copy_zc"]["launches"])

    out = {
        "metric": "migration GB/s (pilot us/prediction; plan us; H2D/D2H vs PCIe Gen5 x16)",
        "value": round(value, 3), "unit": "GB/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(ms_max / args.steps, 3), "higher_is_better": True, "scaling": "weak",
        "instrumented_ms_per_step": round(ms_instr / args.steps, 3),
        "step_bound_ms": round(bound_ms, 3),
        "step_bound_strict_ms": round(bound_strict_ms, 3),
        "step_bound_link_ms": round(bound_fluid_ms, 3),
        "frac_of_link_bound": round(bound_fluid_ms / (ms_max / args.steps), 4) if ms_max else None,
        "frac_of_step_bound": round(bound_ms / (ms_max / args.steps), 4) if ms_max else None,
        "step_bound_note": ("critical path of the timed steps' per-transition H2D / D2H bytes at the probe's "
                            "per-direction rates: EVICT_j (D2H stream, in order) after block j-2; FETCH_j "
                            "after the write-backs overlapping its destination (R21; strict: after the whole "
                            "EVICT_j, R12); block j = ready[j] (no compute emulation) - D2D, plan and pilot "
                            "time not counted; step_bound_link_ms: the same DAG with both directions sharing the "
                            "measured bidirectional aggregate while they overlap (fluid model)"),
        "vs_baseline": None, "dtype": "f32 weights / f64 accumulate (pilot); int64 (plan); u8 (migrate)",
        "data": "synthetic",
        "config": {"workload": args.config, "desc": CONFIG_DESC[args.config], "policy": ("RETAIN" if args.policy & 1 else "PAPER") + ("+SHARE (R20)" if args.policy & 2 else ""),
                   "migrate_order": "R12 strict" if args.strict_order else "R21 per-range",
                   "budget_bytes": wl.budget, "tensors": len(wl.tensors),
                   "l2": "inputs larger than L2 (every step moves >= 1 GiB through HBM and PCIe)",
                   "parallelism": f"{world} independent managers (replicas, no collective on the path)"},
        "compute_emulation": ({"compute_ms_per_step": round(comp_ms_step, 3),
                               "exposed_ms_per_step": round(ms_max / args.steps - comp_ms_step, 3),
                               "exposed_frac_of_compute": round((ms_max / args.steps - comp_ms_step) / comp_ms_step, 4),
                               "compute_only_ms_per_step": round(comp_only_ms, 3),
                               "exposed_vs_compute_only_ms": round(ms_max / args.steps - comp_only_ms, 3),
                               "exposed_vs_compute_only_frac": round((ms_max / args.steps - comp_only_ms) / comp_only_ms, 4),
                               "note": "compute_only = the same spin blocks and per-block event waits with no "
                                       "migrations (the harness's own launch/event cost)"}
                              if emulate else None),
        "pilot_us_per_prediction": round(pred_us, 3),
        "pilot_kernel_us": round(pilot_kernel_us, 3), "decode_kernels_us": round(decode_us, 3),
        "predictions_per_s": round(1e6 / pred_us, 1),
        "pilot_latency_b1": lat,
        "mispredictions": mis,
        "faults": faults,
        "pilot_batch64": {"us_per_batch": round(b64_us, 2), "us_per_prediction": round(b64_us / 64, 3),
                          "predictions_per_s": round(64e6 / b64_us, 1),
                          "pilot_kernel_us": round(b64_kernel_us, 2), "decode_kernels_us": round(b64_decode_us, 2),
                          "kernel": ("pilot_kernel<8> (fp64 DMMA m8n8k4 tensor-core tiles, 8 samples per 16-CTA "
                                     "cluster; north_star gate)" if b64_kern == 0 else "pilot_tc_kernel"),
                          "tensor_roofline": {"bound": "tensor", "achieved": round(tc_flop / (b64_kernel_us * 1e-6) / 1e12, 4),
                                              "peak": round(peaks["bf16_tflops"] * 45.0 / 2250.0, 2), "unit": "TFLOP/s",
                                              "frac": round(tc_flop / (b64_kernel_us * 1e-6) / 1e12 / (peaks["bf16_tflops"] * 45.0 / 2250.0), 5),
                                              "flop_per_launch": tc_flop,
                                              "peak_source": "FP64 tensor = measured bf16 x 45/2250 (guide's nominal B200 ratio)",
                                              "note": "latency-bound: 6 dependent layers"},
                          "tc_opt_in": tc},
        "plan_us": round(plan_us, 2), "transitions_per_step": round(tot_K / args.steps, 2),
        "plan_floor_frac": (round(lat["single_cta_launch_floor_us"] / plan_us, 5)
                            if lat.get("single_cta_launch_floor_us") else None),
        "h2d_bytes_per_step": int(h2d_all / args.steps / world), "d2h_bytes_per_step": int(d2h_all / args.steps / world),
        "pcie": {"h2d_dma_gbs": round(h2d_link, 2) if h2d_link else None,
                 "d2h_dma_gbs": round(d2h_link, 2) if d2h_link else None,
                 "peak_theoretical_gbs": PCIE_GEN5_X16,
                 "probe_h2d_gbs": round(probe["h2d"], 2), "probe_d2h_gbs": round(probe["d2h"], 2),
                 "probe_bidir_gbs": round(bidir, 2),
                 "frac_h2d_of_theoretical": round(h2d_link / PCIE_GEN5_X16, 4) if h2d_link else None,
                 "frac_d2h_of_theoretical": round(d2h_link / PCIE_GEN5_X16, 4) if d2h_link else None,
                 "step_gbs_per_gpu": round(value / world, 3)},
        "roofline": roof,
        "time_shares": shares,
        "mechanisms": ctr,
        "gpu_launches": int(launches),
        "clocks": clk.summary(),
        "host_pool": {"numa_node": host_numa, "gpu_topology": gpu_topology(local),
                      "note": "pinned tensor homes bound to the GPU's NUMA node (mbind before cudaHostRegister; "
                              "-1 = the platform reports no node)"},
        "e2e": {"value": round(bytes_all / e2e_max / 1e9, 3), "unit": "GB/s",
                "h2d_bytes_per_step": int(wl.D_s * 8 + wl.h * 4), "d2h_bytes_per_step": int(16 * 4 + 9 * len(wl.tensors)),
                "note": "dyo_* calls with pinned host sample descriptors; plan lists + residency read back each step"},
    }
    if world == 1 and not args.no_cpu_baseline:
        import os as _os
        b, sec, n = oracle_steps(wl, 200, budget_s=15.0)
        out["cpu_baseline"] = {"value": round(b / sec / 1e9, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                               "sample": f"{n} oracle steps of the same workload (pure Python encode/pilot/decode/plan + "
                                         f"numpy copy of each step's algorithmic bytes), ~15 s, 1 of {_os.cpu_count()} cores"}
        if wl.notes.get("batch", 1) == 1:
            comp = oracle_components(wl)
            out["cpu_baseline"]["components"] = comp
            comp["gpu_speedup"] = {"pilot_decode": round((comp["pilot_us_per_prediction"] + comp["decode_us_per_prediction"])
                                                         / max(pred_us, 1e-9), 1),
                                   "plan": round(comp["plan_us_per_step"] / max(plan_us, 1e-9), 1)}
    d.close()
    if world == 1 and not args.no_cpu_baseline:
        _log("compiled cpu planner")
        try:
            out["cpu_baseline"]["compiled_planner"] = compiled_planner_leg(torch, wl, local, dev_inputs, B, s0, args.steps,
                                                                           plan_us)
        except Exception as e:                  # reported, never fatal to the headline line
            out["cpu_baseline"]["compiled_planner"] = {"error": str(e)[:200]}
    print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


def compiled_planner_leg(torch, wl, dev, inputs, B, s0, n_steps, gpu_plan_us):
    """K2's honest baseline: the compiled single-core CPU planner (baseline/cpu_planner.cpp, g++
    -O3, bit-exact with oracle/plan.py - tests/test_cpu_planner.py) planning the same W sets the GPU
    planner plans. A fresh manager predicts each step on the GPU; its tensor sets are read back
    (untimed), the CPU planner plans them (timed, one host core) and the GPU planner plans them
    too; both start from an empty arena, so every transition's byte counts must agree."""
    import numpy as np
    sys.path.insert(0, os.path.join(ROOT, "baseline"))
    import cpu_planner
    from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo
    # plan-only manager (DYO_F_NO_HOST_POOL = 4): its plans are never migrated, each supersedes the last
    dc = Dyo(wl.budget, wl.align, wl.policy, max_batch=B, device=dev, flags=4)
    dc.load(wl)
    cp = cpu_planner.CpuPlanner(wl)
    n_sites = 4096
    t_cpu, n_tr, mism, steps = 0.0, 0, 0, 0
    for k in range(n_steps):
        desc, hist = inputs(k)
        dc.predict(desc, hist, B, stream=s0.cuda_stream)
        Ws = []
        for b in range(B):
            K, _, _, _ = dc.prediction(b, wl.K_max, n_sites, stream=s0.cuda_stream)
            for g in range(K):
                Ws.append([tuple(int(x) for x in e) for e in dc.group_entries(b, g, cap=1 << 16, stream=s0.cuda_stream)])
        t0 = time.perf_counter()
        st, trs = cp.plan(Ws)
        t_cpu += time.perf_counter() - t0
        K = dc.plan(stream=s0.cuda_stream)
        if st != 0 or K != len(trs):
            mism += 1
            break
        for j in range(K):
            info = dc.plan_info(j)
            if (info["h2d"], info["d2h"], info["d2d"]) != (trs[j]["h2d"], trs[j]["d2h"], trs[j]["d2d"]):
                mism += 1
        n_tr += K
        steps += 1
    torch.cuda.synchronize()
    dc.close()
    cp.close()
    cpu_us = t_cpu / max(1, steps) * 1e6
    return {"plan_us_per_step": round(cpu_us, 1), "transitions_per_step": round(n_tr / max(1, steps), 2),
            "steps": steps, "cores": 1, "transition_mismatches_vs_gpu": mism,
            "gpu_plan_us": round(gpu_plan_us, 2), "gpu_speedup": round(cpu_us / max(gpu_plan_us, 1e-9), 2),
            "sample": "the bench's first %d step inputs, W sets of the GPU decode, planned from an empty arena" % steps,
            "kind": "compiled single-core planner (baseline/cpu_planner.cpp, g++ -O3 -march=x86-64-v3)"}


def gpu_topology(local):
    """This GPU's row of `nvidia-smi topo -m` (GPU <-> GPU / NIC links, CPU and NUMA affinity) and
    its PCIe link, for the multi-manager report (survey §8(e)); None if nvidia-smi is missing."""
    import subprocess
    try:
        topo = subprocess.run(["nvidia-smi", "topo", "-m"], capture_output=True, text=True, timeout=20).stdout
        lines = [ln for ln in topo.splitlines() if ln.strip()]
        head = lines[0].split() if lines else []
        row = next((ln for ln in lines[1:] if ln.split() and ln.split()[0] == f"GPU{local}"), None)
        link = subprocess.run(["nvidia-smi", "-i", str(local), "--query-gpu=pci.bus_id,pcie.link.gen.current,"
                               "pcie.link.width.current", "--format=csv,noheader"],
                              capture_output=True, text=True, timeout=20).stdout.strip()
        return {"header": " ".join(head), "row": " ".join(row.split()) if row else None, "pcie": link}
    except (OSError, subprocess.SubprocessError):
        return None


def step_bound_ms(trs, h2d_gbs, d2h_gbs, strict=False):
    """Lower bound of the migration time of a transition sequence (ms): the dependency DAG of the
    migrate protocol with each direction's DMA at its measured probe rate. EVICT_j runs on the D2H
    stream in order, after block j-2 ended (its half's last user); block j ends when ready[j]
    fires (no emulated compute). R12 (strict, or a transition with compaction MOVEs / > 64
    write-backs / late_all): FETCH_j after the whole EVICT_j. R21 (record detail available): each
    FETCH after block j-2 and the write-backs overlapping its destination; ready[j] after FETCH_j
    and EVICT_j."""
    e_end = 0.0
    f_end = 0.0
    ready = []
    for j, tr in enumerate(trs):
        h2d, d2h = tr[0], tr[1]
        half_free = ready[j - 2] if j >= 2 else 0.0
        relaxed = (not strict and len(tr) > 2 and tr[4] == 0 and not tr[5] and 0 < len(tr[2]) <= 64)
        if not relaxed:
            e_end = max(e_end, half_free) + d2h / (d2h_gbs * 1e6)
            f_end = max(f_end, e_end) + h2d / (h2d_gbs * 1e6)
            ready.append(f_end)
            continue
        t = max(e_end, half_free)
        iv = []
        for src, nb in tr[2]:
            t += nb / (d2h_gbs * 1e6)
            iv.append((src, src + nb, t))
        e_end = t
        f = max(f_end, half_free)
        for dst, nb in tr[3]:
            dep = max([e for lo, hi, e in iv if dst < hi and dst + nb > lo] or [0.0])
            f = max(f, dep) + nb / (h2d_gbs * 1e6)
        # ready[j] joins FETCH_j and EVICT_j; the copy stream itself waits EVICT_j only when the
        # transition has late carries
        f_end = max(f, e_end) if tr[6] else f
        ready.append(max(f, e_end))
    return ready[-1] if ready else 0.0


def step_bound_fluid_ms(trs, h2d_gbs, d2h_gbs, bidir_gbs, strict=False):
    """The record-level DAG of step_bound_ms (the same dependencies: each direction's queue in
    order, EVICT_j after ready[j-2], FETCH_j after the whole EVICT_j (R12) or after the write-backs
    it overwrites (R21), ready[j] after both queues' work of transition j) simulated as a fluid
    model of the PCIe link: each direction alone runs at its probe rate, both at once share the
    measured bidirectional aggregate (in proportion to their solo rates). ms."""
    rh, rd = h2d_gbs * 1e6, d2h_gbs * 1e6                     # bytes per ms
    both = bidir_gbs * 1e6
    bh, bd = min(both * rh / (rh + rd), rh), min(both * rd / (rh + rd), rd)
    tasks, ready_deps = [], []                                 # task: (queue 0 D2H / 1 H2D, bytes, deps)
    last = [None, None]                                        # latest task of each queue so far
    for j, tr in enumerate(trs):
        relaxed = not strict and len(tr) > 2 and tr[4] == 0 and not tr[5] and 0 < len(tr[2]) <= 64
        half = ready_deps[j - 2] if j >= 2 else []
        iv = []
        wbs = tr[2] if len(tr) > 2 else ([(0, tr[1])] if tr[1] else [])
        for src, nb in wbs:
            tasks.append((0, nb, list(half)))
            last[0] = len(tasks) - 1
            iv.append((src, src + nb, last[0]))
        evict_end = [last[0]] if last[0] is not None else []
        fetches = tr[3] if len(tr) > 2 else ([(0, tr[0])] if tr[0] else [])
        for dst, nb in fetches:
            if relaxed:
                dep = [k for lo, hi, k in iv if dst < hi and dst + nb > lo]
                deps = list(half) + dep[-1:]
            else:
                deps = list(half) + evict_end
            tasks.append((1, nb, deps))
            last[1] = len(tasks) - 1
        ready_deps.append(list(half) + [k for k in last if k is not None])
    n = len(tasks)
    rem = [float(t[1]) for t in tasks]
    done = [None] * n
    qs = [[k for k in range(n) if tasks[k][0] == q] for q in (0, 1)]
    head = [0, 0]
    t = 0.0
    while head[0] < len(qs[0]) or head[1] < len(qs[1]):
        run = []
        for q in (0, 1):
            if head[q] < len(qs[q]):
                k = qs[q][head[q]]
                if all(done[d] is not None for d in tasks[k][2]):
                    run.append((q, k))
        if not run:
            return float("nan")          # cannot happen: dependencies point backwards
        two = len(run) == 2
        rate = {0: bd if two else rd, 1: bh if two else rh}
        dt = min(rem[k] / rate[q] for q, k in run)
        t += dt
        for q, k in run:
            rem[k] -= dt * rate[q]
            if rem[k] <= 1e-6:
                done[k] = t
                head[q] += 1
    return max([t for t in done if t is not None] or [0.0])


def bidir_probe(torch, nbytes=256 << 20, reps=3):
    """Aggregate GB/s of one H2D and one D2H copy running at once (two streams)."""
    h1 = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    h2 = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d1 = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    d2 = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s1)
    s2.wait_event(a)
    for _ in range(reps):
        with torch.cuda.stream(s1):
            d1.copy_(h1, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
    s1.wait_stream(s2)
    b.record(s1)
    b.synchronize()
    return 2 * nbytes * reps / (a.elapsed_time(b) * 1e-3) / 1e9


def _log(msg):
    if os.environ.get("DYO_BENCH_VERBOSE"):
        print(f"[bench {time.strftime('%H:%M:%S')}] {msg}", file=sys.stderr, flush=True)


def copy_stamp_report(st, path):
    """Per-launch anatomy of the record-copy kernel in the timed region (DYO_COPY_STAMPS=1): CTA
    start skew, record-scan time, per-CTA copy time and the launch span they add up to."""
    import numpy as np
    if len(st) == 0:
        return None
    cta = ((st[:, 0] >> np.uint64(8)) & np.uint64(0xFFFFFF)).astype(np.int64)
    mk = st[cta == 0xFFF]            # DYO_COPY_STAMPS=2 marker kernels around each launch
    st = st[cta != 0xFFF]
    lid = (st[:, 0] >> np.uint64(32)).astype(np.int64)
    sm = (st[:, 0] & np.uint64(255)).astype(np.int64)
    marks = {}
    for row in mk:
        marks[(int(row[0] >> np.uint64(32)), int(row[0] & np.uint64(255)))] = int(row[1])
    t0, t1, t2 = (st[:, k].astype(np.int64) for k in (1, 2, 3))
    rows = []
    for L in np.unique(lid):
        m = lid == L
        a0, a1, a2 = t0[m], t1[m], t2[m]
        rows.append({"ctas": int(m.sum()), "span_us": (a2.max() - a0.min()) / 1e3,
                     "start_skew_us": (a0.max() - a0.min()) / 1e3, "scan_us_max": (a1 - a0).max() / 1e3,
                     "cta_copy_us_med": float(np.median(a2 - a1)) / 1e3, "cta_copy_us_max": (a2 - a1).max() / 1e3,
                     "end_skew_us": (a2.max() - a2.min()) / 1e3, "distinct_sms": int(len(np.unique(sm[m])))})
        if (int(L), 0) in marks and (int(L), 1) in marks:
            rows[-1]["mark_to_first_cta_us"] = (a0.min() - marks[(int(L), 0)]) / 1e3
            rows[-1]["last_cta_to_mark_us"] = (marks[(int(L), 1)] - a2.max()) / 1e3
    keys = [k for k in rows[0].keys() if all(k in r for r in rows)]
    med = {k: float(np.median([r[k] for r in rows])) for k in keys}
    big = [r for r in rows if r["span_us"] >= 20]
    out = {"launches": len(rows), "median": med, "sum_span_us": float(sum(r["span_us"] for r in rows)),
           "mean_span_us": float(np.mean([r["span_us"] for r in rows])),
           "median_over_launches_ge_20us": {k: float(np.median([r[k] for r in big])) for k in keys} if big else None,
           "first_20": rows[:20]}
    if path:
        os.makedirs(os.path.dirname(path) or ".", exist_ok=True)
        with open(path, "w") as f:
            json.dump(out, f, indent=1)
    return out


def main():
    args = parse()
    wd = os.environ.get("DYO_BENCH_WATCHDOG")
    if wd:
        import faulthandler
        faulthandler.dump_traceback_later(float(wd), exit=True)
    if args.impl == "reference":
        run_reference(args)
    else:
        run_dyo(args)


if __name__ == "__main__":
    main()
