"""PyTorch integration measured (survey §8(f) rank 3): the real Tree-LSTM of
paper_conf_hpca_renxyzlnwxl24_b200.torch_runtime trained with libdyo-managed tensors vs all
tensors resident (plain PyTorch): wall time per step (exposed = the difference), faults, and the
largest batch each fits under a device budget (resident: every tensor of the batch on the device;
libdyo: every block's tensor set within half the budget - dyo_plan feasibility)."""
import json, os, sys, time
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch
import workloads as WL
from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo, DyoError
from paper_conf_hpca_renxyzlnwxl24_b200.torch_runtime import TreeLSTMRuntime

out = {}
budget = 48 << 20
for B in (4, 16):
    wl = WL.make("tree", n_samples=64, batch=B, budget=budget)
    res = {}
    for mode in ("resident", "dyo"):
        rt = TreeLSTMRuntime(wl, mode=mode)
        rt.step(list(range(B)))                       # warm-up
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        n = 3
        for s in range(1, 1 + n):
            rt.step([(s * B + i) % 64 for i in range(B)])
        torch.cuda.synchronize()
        res[mode] = (time.perf_counter() - t0) * 1e3 / n
        rt.close()
        if mode == "dyo":
            res["faults_total"] = rt.faults
    out[f"B={B}"] = {"ms_per_step_resident": round(res["resident"], 2), "ms_per_step_dyo": round(res["dyo"], 2),
                     "overhead_frac": round(res["dyo"] / res["resident"] - 1, 4), "faults": res["faults_total"]}

# largest batch under the budget
wl64 = WL.make("tree", n_samples=64, batch=64, budget=budget)
per_sample = sum(t.nbytes for t in wl64.tensors if t.name.startswith(("h[0,", "c[0,", "g[0,", "x[0,")))
shared = sum(t.nbytes for t in wl64.tensors if "[" not in t.name or t.name.startswith(("Wh", "gWh")))
res_max = max(0, (budget - shared) // per_sample)
d = Dyo(budget, 256, 1, max_batch=64, flags=4)
d.load(wl64)
dyo_max = 0
hist = np.tile(wl64.hist_ids.astype(np.int32), (64, 1))
for B in (1, 2, 4, 8, 16, 32, 64):
    try:
        d.predict(wl64.samples[:B].copy(), hist[:B], B)
        d.plan()
        dyo_max = B
    except DyoError:
        break
d.close()
out["max_batch"] = {"budget_mib": budget >> 20, "resident_max_batch": int(res_max), "dyo_max_batch_tested": dyo_max,
                    "note": "resident: shared weights/grads + per-sample node tensors all on the device; libdyo: every "
                            "block's tensor set within half the budget (dyo_plan feasible); tested up to the workload's 64"}
print(json.dumps(out))
