"""Per-tile timeline (SM cycles, CTA 0) of the stem halo kernel as the bench runs it (QC_DEBUG
build, QC_TRACE).  Usage: python scripts/trace_stem.py out.bin [bits] [layer_index]"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
out = sys.argv[1]
os.environ["QC_TRACE"] = out
if os.path.exists(out):
    os.remove(out)
import torch  # noqa: E402
import bench  # noqa: E402

bits = int(sys.argv[2]) if len(sys.argv) > 2 else 4
j = int(sys.argv[3]) if len(sys.argv) > 3 else 0
os.environ.pop("QC_TRACE")
from paper_conf_icpp_hanhyylhgwwlq20_b200 import tuning  # noqa: E402
tuning.load_plans(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "plans",
                               f"resnet50_trunk_a{bits}_b256.json"))
tr = bench.Trunk(bits, 256, torch.device("cuda", 0))
torch.cuda.synchronize()
os.environ["QC_TRACE"] = out
L = tr.layers[j]
print(L["name"], L["plan"])
for _ in range(2):
    if j == 0:
        tr.qc.qconv2d_forward_quantize(L["desc"], tr.x_float, tr.s_in, L["w"], L["bias"], L["m"], L["n"], y=L["y"])
    else:
        tr.qc.qconv2d_forward(L["desc"], L["x"], L["w"], L["bias"], L["m"], L["n"], y=L["y"])
torch.cuda.synchronize()
t = np.fromfile(out, dtype=np.uint64).reshape(-1, 16, 1024).astype(np.int64)[-1]
t0 = min(v for v in t.reshape(-1) if v > 0)
names = {0: "prod", 2: "mma_acc_free", 3: "mma_in", 1: "mma_fenced", 11: "mma_issued", 12: "commit_empty",
         4: "commit_tfull", 5: "epi_acc_full", 6: "epi_done", 7: "store", 8: "cvt_in", 10: "epi_stg_free", 13: "epi_ld_done", 14: "epi_requant_done", 9: "cvt_done"}
if L["plan"]["kernel_name"] not in ("halo", "halo_t"):
    names = {i: f"ev{i}" for i in range(16)}
for ev, nm in names.items():
    row = t[ev][t[ev] > 0] - t0
    if len(row) > 1:
        print(f"{nm:14s} n={len(row):4d} first {row[:8].tolist()} mean dt {np.diff(row[:200]).mean():.0f}")
