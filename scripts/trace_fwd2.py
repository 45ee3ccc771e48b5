"""Timeline of the first CTA pair of the CTA-pair kernel for one trunk layer (debug; QC_TRACE + QC_CTA2)."""
import os, sys
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
bits, out, name = int(sys.argv[1]), sys.argv[2], sys.argv[3]
import torch
import bench
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc
tr = bench.Trunk(bits, 256, "cuda")
L = next(l for l in tr.layers if l["name"] == name)
if os.path.exists(out): os.remove(out)
qc.qconv2d_forward(L["desc"], L["x"], L["w"], L["bias"], L["m"], L["n"], y=L["y"])
torch.cuda.synchronize()
t = np.fromfile(out, dtype=np.uint64).reshape(-1, 16, 1024).astype(np.int64)
t = t.max(axis=0)   # both CTAs' dumps: union of the written slots
t0 = min(v for v in t.reshape(-1) if v > 0)
names = {0: "prod0_issue", 7: "prod1_issue", 2: "mma_wait_start", 3: "mma_stage_done", 5: "cvt0_full", 6: "cvt0_done", 8: "cvt1_full", 9: "cvt1_done"}
for ev, nm in names.items():
    row = t[ev]; row = row[row > 0] - t0
    if len(row) > 1:
        print(f"{nm:16s} n={len(row):4d} first={row[:6].tolist()} med_gap={np.median(np.diff(row)):.0f}")
