"""Planner phase stamps (clock64 cycles) of transition J of a plan, plus the per-plan time by
kernel kind: python tools/prof_plan.py <cfg> <B> <J>..."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import workloads as WL
from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo
cfg = sys.argv[1] if len(sys.argv) > 1 else "moe"
B = int(sys.argv[2]) if len(sys.argv) > 2 else 1
Js = [int(x) for x in sys.argv[3:]] or [3]
POL = int(os.environ.get("PLAN_POLICY", "-1"))
wl = WL.make(cfg, n_samples=max(64, B))
d = Dyo(wl.budget, wl.align, wl.policy if POL < 0 else POL, max_batch=B, flags=4 | 8)
d.load(wl)
s = torch.cuda.current_stream().cuda_stream
desc = torch.from_numpy(wl.samples.copy()).cuda()
hist = torch.from_numpy(np.tile(wl.hist_ids.astype(np.int32), (B, 1))).cuda() if wl.h else None
names = ["start", "A W_j/need", "B scan", "C select", "D kept/evict+gaps", "E place order", "first fit+compact",
         "F records/state", "G rebuild"]
for step in range(3):
    for J in Js:
        d.predict(desc[(step * B) % 64:(step * B) % 64 + B], hist, B, stream=s)
        d.plan_stamps(J)
        d.timings(reset=True)
        d.plan(stream=s)
        tm = d.timings(reset=True)
        st = d.plan_stamps(-1).astype(np.int64)
        dif = {names[i]: int(st[i] - st[i - 1]) for i in range(1, 9) if st[i] > 0 and st[i - 1] > 0}
        info = d.plan_info(J) if J < d.K else {}
        print(f"{cfg} step {step}: plan {tm['plan']['ms'] * 1e3:.1f} us; K {d.K}; transition {J} "
              f"(ent {info.get('n_entries')}, ev {info.get('n_evict')}, mv {info.get('n_move')}, ca {info.get('n_carry')}, "
              f"al {info.get('n_alloc')}, fe {info.get('n_fetch')}) cycles:", dif, "total", int(st[8] - st[0]) if st[8] else None,
              f"nm {st[60]} ng {st[61]} kept {st[62]} regmode {st[63]}")
