"""Time every candidate plan of one conv shape (8-bit, seeded codes): python scripts/cand_shape.py
n h w c k r s stride pad [bits]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc  # noqa: E402
import workloads as W  # noqa: E402

n, h, w, c, k, r, s, st, pad = map(int, sys.argv[1:10])
bits = int(sys.argv[10]) if len(sys.argv) > 10 else 8
cs = W.ConvShape("x", n, h, w, c, k, r, s, st, pad)
li = W.make_layer_inputs(cs, bits, seed=1)
m, sh = qc.qconv_requant_params(li.s_x, li.s_w, li.s_y)
d = qc.make_desc(n, h, w, c, k, r, s, stride=st, pad=pad, x_t=li.x_t, w_t=li.w_t, y_t=li.y_t,
                 clamp_lo=li.clamp_lo, clamp_hi=li.clamp_hi)
x = torch.from_numpy(li.x_bytes).cuda()
wt = torch.from_numpy(li.w_bytes).cuda()
b, mm, nn = (torch.from_numpy(a).cuda() for a in (li.bias, m, sh))
res = []
for cand in [None] + qc.qconv_plan_candidates(d):
    if cand is not None:
        qc.qconv_plan_set(d, cand["kernel"], cand["bn"])
    plan = qc.qconv_debug_plan(d)
    for _ in range(3):
        qc.qconv2d_forward(d, x, wt, b, mm, nn)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10):
        qc.qconv2d_forward(d, x, wt, b, mm, nn)
    e1.record()
    torch.cuda.synchronize()
    res.append((round(e0.elapsed_time(e1) / 10 * 1e3, 1), "default" if cand is None else "", plan["kernel_name"], plan["bn"], plan.get("prologue")))
qc.qconv_plan_set(d, None)
for r_ in sorted(res):
    print(r_)
