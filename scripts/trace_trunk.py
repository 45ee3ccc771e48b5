"""Pipeline timeline of CTA 0 for chosen layers of the bench trunk (QC_TRACE; debug only).

usage: python scripts/trace_trunk.py BITS out.bin layer [layer ...]
Prints, per layer, the median gap between consecutive events of each kind and the
producer->consumer latency of each ring stage (TMA issue -> data landed)."""
import os, sys
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
bits, out = int(sys.argv[1]), sys.argv[2]
names = sys.argv[3:]
import torch
import bench
tr = bench.Trunk(bits, 256, "cuda")
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc
EV = ["prod_issue", "mma_fenced", "mma_tempty_ok", "mma_full_ok", "mma_commit", "epi_tfull_ok", "epi_tempty_arrive",
      "epi_store_issued", "cvt_full_ok", "cvt_done", "cvt_loop_done", "mma_issued", "mma_commit1"]
for L in tr.layers:
    if L["name"] not in names:
        continue
    for _ in range(2):
        qc.qconv2d_forward(L["desc"], L["x"], L["w"], L["bias"], L["m"], L["n"], y=L["y"])
    torch.cuda.synchronize()
    os.environ["QC_TRACE"] = out
    if os.path.exists(out):
        os.remove(out)
    # QC_TRACE is read once per process by the library: this script must be started with it set
    qc.qconv2d_forward(L["desc"], L["x"], L["w"], L["bias"], L["m"], L["n"], y=L["y"])
    torch.cuda.synchronize()
    if not os.path.exists(out):
        print("no trace written (start with QC_TRACE set)"); break
    t = np.fromfile(out, dtype=np.uint64).reshape(-1, 16, 1024).astype(np.int64)[-1]
    t0 = min(v for v in t.reshape(-1) if v > 0)
    print(f"== {L['name']} ({bits}-bit)")
    for ev, nm in enumerate(EV):
        row = t[ev]
        row = row[row > 0] - t0
        if len(row) > 1:
            print(f"  {nm:18s} n={len(row):4d} first={row[:5].tolist()} med_gap={np.median(np.diff(row)):.0f} ns last={row[-1]}")
    issue = t[0][t[0] > 0] - t0
    landed = (t[8] if (t[8] > 0).any() else t[3])
    landed = landed[landed > 0] - t0
    n = min(len(issue), len(landed))
    if n > 4:
        lat = landed[:n] - issue[:n]
        print(f"  stage latency issue->landed-seen: median {np.median(lat):.0f} ns  p90 {np.percentile(lat, 90):.0f} ns")
