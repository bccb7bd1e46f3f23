"""Planner phase stamps (clock64 cycles) for one transition of the MoE / AF plans."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import workloads as WL
from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo
cfg = sys.argv[1] if len(sys.argv) > 1 else "moe"
wl = WL.make(cfg, n_samples=64)
d = Dyo(wl.budget, wl.align, wl.policy, max_batch=1, flags=4 | 8)
d.load(wl)
s = torch.cuda.current_stream().cuda_stream
desc = torch.from_numpy(wl.samples.copy()).cuda()
hist = torch.from_numpy(wl.hist_ids.astype(np.int32).reshape(1, -1)).cuda() if wl.h else None
names = ["start", "A load/need", "B", "C classify", "D candidates", "E retain", "F evict recs", "G kept", "H gaps",
         "I place order", "J first fit", "compaction", "K records", "L state", "pw/next", "res lists", "M header"]
for step in range(4):
    d.predict(desc[step:step + 1], hist, 1, stream=s)
    d.plan_stamps(3)
    d.timings(reset=True)
    d.plan(stream=s)
    tm = d.timings(reset=True)
    st = d.plan_stamps(-1).astype(np.int64)
    dif = {names[i]: int(st[i] - st[i - 1]) for i in range(1, 16) if st[i] > 0 and st[i - 1] > 0}
    print(f"{cfg} step {step}: plan {tm['plan']['ms'] * 1e3:.1f} us;", "transition 3 phase cycles:", dif, "total", int(st[15] - st[0]) if st[15] else None)
