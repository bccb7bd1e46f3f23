"""K1-TC phase stamps (globaltimer ns, CTA 0) and latency for a batch of B predictions."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import workloads as WL
from paper_conf_hpca_renxyzlnwxl24_b200 import Dyo
cfg = sys.argv[1] if len(sys.argv) > 1 else "moe"
B = int(sys.argv[2]) if len(sys.argv) > 2 else 64
wl = WL.make(cfg, n_samples=max(64, B))
d = Dyo(wl.budget, wl.align, wl.policy, max_batch=B, flags=4 | 8 | 32)   # 32: DYO_F_PILOT_TC
d.load(wl)
s = torch.cuda.current_stream()
desc = torch.from_numpy(wl.samples[:B].copy()).cuda()
hist = torch.from_numpy(np.tile(wl.hist_ids.astype(np.int32), (B, 1))).cuda() if wl.h else None
for i in range(3):
    d.predict(desc, hist, B, stream=s.cuda_stream)
d.pilot_stamps(True)
d.predict(desc, hist, B, stream=s.cuda_stream)
st = d.pilot_stamps(False).astype(np.int64)
t0 = st[0]
rel = lambda i: (st[i] - t0) / 1e3 if st[i] >= t0 else None
print(f"{cfg} B={B} stamps (us from kernel start): init {rel(1)}, features {rel(2)}")
for k in range(8):
    print(f"  stage {k}: X full {rel(3 + k)}  D ready {rel(11 + k)}  prog {rel(19 + k) if k < 8 else None}")
print(f"  end {rel(27)}; stage 1 detail: before redfull {rel(28)}, redfull done {rel(29)}, before prog arrive {rel(30)}, reduce done e0 {rel(31)} e96 {rel(26)}")
