import sys, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc, oracle, workloads as W
for name in ["res2a_branch2c", "res2a_branch2a", "res3a_branch2c"]:
  for bits in (8, 4):
    cs = next(c for c in W.resnet50_convs(2) if c.name == name)
    li = W.make_layer_inputs(cs, bits, seed=3)
    m, n = qc.qconv_requant_params(li.s_x, li.s_w, li.s_y)
    d = qc.make_desc(cs.n, cs.h, cs.w, cs.c, cs.k, cs.r, cs.s, stride=cs.stride, pad=cs.pad, x_t=li.x_t, w_t=li.w_t, y_t=li.y_t, clamp_lo=li.clamp_lo, clamp_hi=li.clamp_hi)
    L = qc.QConv2d.create(d, li.w_bytes, li.bias, m, n, device="cuda")
    y = L(torch.from_numpy(li.x_bytes).cuda()).cpu().numpy()
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    bad = np.argwhere(y.reshape(-1, y.shape[-1]) != ref.reshape(-1, ref.shape[-1]))
    print(name, bits, qc.qconv_debug_plan(d)['kernel_name'], qc.qconv_debug_plan(d)['bn'], "mismatch rows/cols:", len(bad), bad[:6].tolist())
