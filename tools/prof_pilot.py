"""Focused driver for profiling the pilot path: N back-to-back predictions of a config."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import workloads as WL
from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo

cfg = sys.argv[1] if len(sys.argv) > 1 else "moe"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 50
B = int(sys.argv[3]) if len(sys.argv) > 3 else 1
wl = WL.make(cfg, n_samples=64)
d = Dyo(wl.budget, wl.align, wl.policy, max_batch=B, flags=4 | 8)
d.load(wl)
s = torch.cuda.current_stream()
desc = torch.from_numpy(wl.samples.copy()).cuda()
hist = torch.from_numpy(np.tile(wl.hist_ids.astype(np.int32), (B, 1))).cuda() if wl.h else None
for i in range(5):
    d.predict(desc[:B], hist, B, stream=s.cuda_stream)
torch.cuda.synchronize()
d.timings(reset=True)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(s)
t0 = time.perf_counter()
for i in range(n):
    d.predict(desc[(i % 32):(i % 32) + B], hist, B, stream=s.cuda_stream)
e1.record(s)
e1.synchronize()
t1 = time.perf_counter()
tm = d.timings(reset=True)
d.pilot_stamps(True)
for i in range(3):
    d.predict(desc[:B], hist, B, stream=s.cuda_stream)
st = d.pilot_stamps(False).astype(np.int64)
base = st[0]
sd = {i: int(st[i] - base) for i in range(30) if st[i] >= base and st[i] - base < 10**8}
print("prologue", sd.get(1), sd.get(2), "| stage (wait_in, wait_w, compute):",
      [(sd.get(3 + 3 * k, 0) - (sd.get(2) if k == 0 else sd.get(2 + 3 * k, 0)), sd.get(4 + 3 * k, 0) - sd.get(3 + 3 * k, 0),
        sd.get(5 + 3 * k, 0) - sd.get(4 + 3 * k, 0)) for k in range(7) if (3 + 3 * k) in sd],
      "| head: counts, branch, pieces, cut:", sd.get(21, 0) - sd.get(30, 0), sd.get(22, 0) - sd.get(21, 0), sd.get(23, 0) - sd.get(22, 0), sd.get(26, 0) - sd.get(23, 0),
      "| group: rows, scan, records:", sd.get(24, 0) - sd.get(26, 0), sd.get(25, 0) - sd.get(24, 0), sd.get(31, 0) - sd.get(25, 0), "rest", sd.get(27, 0) - sd.get(31, 0),
      "| epilogue: csync, tables, logits:", sd.get(28, 0) - sd.get(20, 0), sd.get(29, 0) - sd.get(28, 0), sd.get(30, 0) - sd.get(29, 0),
      "| decode head, groups:", sd.get(26, 0) - max([v for k2, v in sd.items() if k2 < 26] or [0]), sd.get(27, 0) - sd.get(26, 0))
print("raw (stamp: cycles since 0):", sorted(sd.items(), key=lambda kv: kv[1]))
print(f"{cfg} B={B}: {e0.elapsed_time(e1) * 1e3 / n:.2f} us/predict (device span), host {(t1 - t0) * 1e6 / n:.2f} us/call, "
      f"pilot event {tm['pilot']['ms'] * 1e3 / max(1, tm['pilot']['launches']):.2f} us, decode event "
      f"{tm['decode']['ms'] * 1e3 / max(1, tm['decode']['launches']):.2f} us")
