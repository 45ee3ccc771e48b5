"""Time chosen layers of the bench trunk (CUDA events, 20 launches each; debug/experiments).
usage: python scripts/time_trunk.py BITS layer [layer ...]   (QC_EXPERIMENT=<flags> for ablations)"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc
bits = int(sys.argv[1])
tr = bench.Trunk(bits, 256, "cuda")
for L in tr.layers:
    if L["name"] not in sys.argv[2:] and "all" not in sys.argv[2:]:
        continue
    f = lambda: qc.qconv2d_forward(L["desc"], L["x"], L["w"], L["bias"], L["m"], L["n"], y=L["y"])
    for _ in range(3): f()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20): f()
    e1.record(); torch.cuda.synchronize()
    us = e0.elapsed_time(e1) / 20 * 1e3
    print(f"{L['name']:18s} {bits}-bit {us:8.1f} us {L['ops'] / us / 1e6:8.1f} TOPS exp={os.environ.get('QC_EXPERIMENT', '0')}")
