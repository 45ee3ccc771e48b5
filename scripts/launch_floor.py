"""Latency floor of one launch under the per-layer bench conditions (L2 flushed, CUDA events):
an empty torch kernel, a 1-element torch op, and our conv kernels on a 1-tile problem."""
import os, statistics, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc
import workloads as W
dev = torch.device("cuda", 0)
flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
def t(fn, n=30, fl=True):
    for _ in range(5): fn()
    ts = []
    for i in range(n):
        if fl: flush.fill_(i & 255)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); ts.append((a, b))
    torch.cuda.synchronize()
    return statistics.median(x.elapsed_time(y) * 1e3 for x, y in ts)
z = torch.zeros(1, device=dev)
print("torch add_ 1 elem, flushed", t(lambda: z.add_(1)))
print("torch add_ 1 elem, warm", t(lambda: z.add_(1), fl=False))
for name, cs, bits, kern in [("1x1 tiny", W.ConvShape("a", 1, 8, 16, 64, 64, 1, 1), 8, None),
                             ("3x3 tiny", W.ConvShape("b", 1, 8, 16, 64, 64, 3, 3, 1, 1), 8, None),
                             ("C1", W.C1, 8, None)]:
    lp = W.make_layer_params(cs, bits, 1)
    d = qc.make_desc(cs.n, cs.h, cs.w, cs.c, cs.k, cs.r, cs.s, stride=cs.stride, pad=cs.pad, relu=True)
    w = qc.qconv_prepare_weights(d, torch.from_numpy(np.ascontiguousarray(lp.w_bytes)).to(dev)); d.w_prepared = 1
    m, n = qc.qconv_requant_params(lp.s_x, lp.s_w, lp.s_y)
    b, mm, nn = (torch.from_numpy(v).to(dev) for v in (lp.bias, m, n))
    x = W.device_post_relu_codes((cs.n, cs.h, cs.w, cs.c), bits, 3, dev)
    y = qc.qconv2d_forward(d, x, w, b, mm, nn)
    f = lambda: qc.qconv2d_forward(d, x, w, b, mm, nn, y=y)
    for kname, kk in [("default", None)] + [(c["kernel_name"] + "/" + str(c["bn"]), c) for c in qc.qconv_plan_candidates(d)]:
        if kk is not None: qc.qconv_plan_set(d, kk["kernel"], kk["bn"])
        print(f"{name:10s} {kname:14s} flushed {t(f):6.1f} us  warm {t(f, fl=False):6.1f} us  plan {qc.qconv_debug_plan(d)['stages']} stages {qc.qconv_debug_plan(d)['smem_bytes']} B")
        qc.qconv_plan_set(d, None)
