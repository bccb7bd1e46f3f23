"""Isolated D2D copy bandwidth of the library's SM and TMA segment-copy kernels (read+write bytes)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import workloads as WL
from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo
wl = WL.make("tiny")
d = Dyo(wl.budget, flags=4)
d.load(wl)
s = torch.cuda.current_stream()
for nb in (64 << 20, 1 << 30):
    a = torch.empty(nb, dtype=torch.uint8, device="cuda"); b = torch.empty(nb, dtype=torch.uint8, device="cuda")
    for mode in (0, 1):
        d.debug_copy(a.data_ptr(), b.data_ptr(), nb, mode, s.cuda_stream)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(5):
            d.debug_copy(a.data_ptr(), b.data_ptr(), nb, mode, s.cuda_stream)
        e1.record(s); e1.synchronize()
        ms = e0.elapsed_time(e1) / 5
        print(f"{'TMA' if mode else 'SM '} {nb >> 20} MiB: {2 * nb / ms / 1e6:.0f} GB/s (r+w) incl. descriptor upload")
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s); b.copy_(a); e1.record(s); e1.synchronize()
    print(f"torch copy_ {nb >> 20} MiB: {2 * nb / e0.elapsed_time(e1) / 1e6:.0f} GB/s")
