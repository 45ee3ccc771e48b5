"""Time every candidate plan of chosen trunk layers (batch 256, bench inputs, L2 not flushed):
python scripts/cand_times.py bits layer [layer ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import bench  # noqa: E402

bits = int(sys.argv[1])
tr = bench.Trunk(bits, 256, torch.device("cuda", 0))
qc = tr.qc
for j in map(int, sys.argv[2:]):
    L = tr.layers[j]
    d = L["desc"]
    res = []
    for c in qc.qconv_plan_candidates(d):
        qc.qconv_plan_set(d, c["kernel"], c["bn"])
        for _ in range(3):
            qc.qconv2d_forward(d, L["x"], L["w"], L["bias"], L["m"], L["n"], y=L["y"])
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(20):
            qc.qconv2d_forward(d, L["x"], L["w"], L["bias"], L["m"], L["n"], y=L["y"])
        e1.record()
        torch.cuda.synchronize()
        res.append((round(e0.elapsed_time(e1) / 20 * 1e3, 1), c["kernel_name"], c["bn"]))
    qc.qconv_plan_set(d, None)
    print(L["name"], sorted(res))
