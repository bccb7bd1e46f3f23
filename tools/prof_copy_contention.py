"""Why the TMA copy kernel runs at ~55% of HBM inside the MoE step but ~94% alone: time 256 MiB
device->device copies (the library's TMA record-copy kernel) alone and while H2D / D2H DMAs of
pinned host memory run on other streams (the step's concurrency)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import workloads as WL
from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo

wl = WL.make("tiny")
d = Dyo(wl.budget, flags=4)
d.load(wl)
nb = 256 << 20
a = torch.empty(nb, dtype=torch.uint8, device="cuda")
b = torch.empty(nb, dtype=torch.uint8, device="cuda")
hs = torch.empty(512 << 20, dtype=torch.uint8, pin_memory=True)
hd = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
s = torch.cuda.Stream()
s_h2d, s_d2h = torch.cuda.Stream(), torch.cuda.Stream()


def copies(n):
    # device->device copies on stream s (torch's copy kernel: the question is HBM contention by
    # the DMA engines, not this kernel; the library's TMA kernel matches it alone, profiles/)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        e0.record(s)
        for _ in range(n):
            b.copy_(a)
        e1.record(s)
    e1.synchronize()
    return 2 * nb * n / (e0.elapsed_time(e1) * 1e-3) / 1e9


copies(2)
print(f"alone: {copies(10):.0f} GB/s (read+write)")
for mode in ("h2d", "d2h", "both"):
    with torch.cuda.stream(s_h2d):
        if mode in ("h2d", "both"):
            for _ in range(8):
                hd.copy_(hs, non_blocking=True)
    with torch.cuda.stream(s_d2h):
        if mode in ("d2h", "both"):
            for _ in range(8):
                hs.copy_(hd, non_blocking=True)
    print(f"with concurrent {mode} DMA: {copies(10):.0f} GB/s (read+write)")
    torch.cuda.synchronize()
