"""Batch-64 pilot sweep: device time per launch of the default K1 batch path (fp64 DMMA tiles)
for the cluster sizes in DYO_PILOT_BATCH_C, plus the max active clusters per size.
Run one process per cluster size (the override is read once): python tools/sweep_batch_pilot.py <cfg>"""
import os, sys, json
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np, torch
import workloads as WL
from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo

cfg = sys.argv[1] if len(sys.argv) > 1 else "moe"
B = int(sys.argv[2]) if len(sys.argv) > 2 else 64
wl = WL.make(cfg, n_samples=max(64, B))
d = Dyo(wl.budget, wl.align, wl.policy, max_batch=B, flags=4 | 8 | int(os.environ.get("EXTRA_FLAGS", "0")))
d.load(wl)
desc = torch.from_numpy(wl.samples[:B].copy()).cuda()
hist = torch.from_numpy(np.tile(wl.hist_ids.astype(np.int32), (B, 1))).cuda() if wl.h else None
s = torch.cuda.current_stream().cuda_stream
for _ in range(5):
    d.predict(desc, hist, B, stream=s)
torch.cuda.synchronize()
d.timings(reset=True)
for _ in range(50):
    d.predict(desc, hist, B, stream=s)
torch.cuda.synchronize()
t = d.timings(reset=True)
print(json.dumps({"cfg": cfg, "B": B, "C": os.environ.get("DYO_PILOT_BATCH_C", "auto"), "kernel": d.query("pilot_kernel"),
                  "pilot_us": t["pilot"]["ms"] * 1e3 / t["pilot"]["launches"],
                  "decode_us": t["decode"]["ms"] * 1e3 / max(1, t["decode"]["launches"])}))
