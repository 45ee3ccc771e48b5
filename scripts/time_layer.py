"""Time single conv layers (CUDA events) -- debug/experiments."""
import os, sys, numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc
import workloads as W
for spec in sys.argv[1:]:
    name, bits = spec.split(':'); bits = int(bits)
    cs = next(c for c in W.resnet50_convs(256) if c.name == name)
    c_st = W.stored_channels(cs, bits)
    lp = W.make_layer_params(cs, bits, 1, c_store=c_st)
    xt = W.U4 if bits == 4 else W.U8
    d = qc.make_desc(cs.n, cs.h, cs.w, c_st, cs.k, cs.r, cs.s, stride=cs.stride, pad=cs.pad, x_t=xt, w_t=lp.w_t, y_t=xt, relu=True)
    x = torch.randint(0, 255, (cs.n, cs.h, cs.w, c_st * bits // 8), dtype=torch.uint8, device="cuda")
    w = qc.qconv_prepare_weights(d, torch.from_numpy(lp.w_bytes.reshape(-1).copy()).cuda()); d.w_prepared = 1
    m, n = qc.qconv_requant_params(lp.s_x, lp.s_w, lp.s_y)
    b = torch.from_numpy(lp.bias).cuda(); mm = torch.from_numpy(m).cuda(); nn = torch.from_numpy(n).cuda()
    y = qc.qconv2d_forward(d, x, w, b, mm, nn)
    for _ in range(3): qc.qconv2d_forward(d, x, w, b, mm, nn, y=y)
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20): qc.qconv2d_forward(d, x, w, b, mm, nn, y=y)
    e1.record(); torch.cuda.synchronize()
    us = e0.elapsed_time(e1) / 20 * 1e3
    print(f"{spec:24s} {us:8.1f} us  {2*cs.macs/us/1e6:8.1f} TOPS  exp={os.environ.get('QC_EXPERIMENT','0')}")
