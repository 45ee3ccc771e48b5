"""Run one trunk layer of the bench (default: the fused fp32 stem) a few times -- a target for
ncu captures of a single kernel.  Usage: python scripts/run_layer.py [bits] [layer] [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import bench  # noqa: E402

bits = int(sys.argv[1]) if len(sys.argv) > 1 else 4
j = int(sys.argv[2]) if len(sys.argv) > 2 else 0
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
from paper_conf_icpp_hanhyylhgwwlq20_b200 import tuning  # noqa: E402
tuning.load_plans(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "plans",
                               f"resnet50_trunk_a{bits}_b256.json"))
tr = bench.Trunk(bits, 256, torch.device("cuda", 0))
L = tr.layers[j]
print(L["name"], L["plan"])
for _ in range(reps):
    if j == 0:
        tr.qc.qconv2d_forward_quantize(L["desc"], tr.x_float, tr.s_in, L["w"], L["bias"], L["m"], L["n"], y=L["y"])
    else:
        tr.qc.qconv2d_forward(L["desc"], L["x"], L["w"], L["bias"], L["m"], L["n"], y=L["y"])
torch.cuda.synchronize()
