"""Planner phase stamps (clock64 cycles) for one transition of the MoE / AF plans."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import workloads as WL
from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo
cfg = sys.argv[1] if len(sys.argv) > 1 else "moe"
B = int(sys.argv[2]) if len(sys.argv) > 2 else 1
J = int(sys.argv[3]) if len(sys.argv) > 3 else 3
wl = WL.make(cfg, n_samples=max(64, B))
d = Dyo(wl.budget, wl.align, wl.policy, max_batch=B, flags=4 | 8)
d.load(wl)
s = torch.cuda.current_stream().cuda_stream
desc = torch.from_numpy(wl.samples.copy()).cuda()
hist = torch.from_numpy(np.tile(wl.hist_ids.astype(np.int32), (B, 1))).cuda() if wl.h else None
names = ["start", "A load/need", "B", "C classify", "D candidates", "E retain", "F evict recs", "G kept", "H gaps",
         "I place order", "J first fit", "compaction", "K records", "L state", "pw/next", "res lists", "M header"]
for step in range(4):
    d.predict(desc[step:step + B], hist, B, stream=s)
    d.plan_stamps(J)
    d.timings(reset=True)
    d.plan(stream=s)
    tm = d.timings(reset=True)
    st = d.plan_stamps(-1).astype(np.int64)
    dif = {names[i]: int(st[i] - st[i - 1]) for i in range(1, 16) if st[i] > 0 and st[i - 1] > 0}
    print(f"{cfg} step {step}: plan {tm['plan']['ms'] * 1e3:.1f} us;", f"transition {J} phase cycles:", dif, "total", int(st[15] - st[0]) if st[15] else None)
