"""Run one conv layer with QC_TRACE set and print CTA 0's pipeline timeline (debug)."""
import os, sys, numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
out = sys.argv[1]
os.environ["QC_TRACE"] = out
if os.path.exists(out): os.remove(out)
import torch
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc
import workloads as W
for name, bits in [(a, int(b)) for a, b in (s.split(':') for s in sys.argv[2:])]:
    cs = next(c for c in W.resnet50_convs(256) if c.name == name)
    c_st = W.stored_channels(cs, bits)
    lp = W.make_layer_params(cs, bits, 1, c_store=c_st)
    xt = W.U4 if bits == 4 else W.U8
    d = qc.make_desc(cs.n, cs.h, cs.w, c_st, cs.k, cs.r, cs.s, stride=cs.stride, pad=cs.pad, x_t=xt, w_t=lp.w_t, y_t=xt, relu=True)
    x = torch.randint(0, 255, (cs.n, cs.h, cs.w, c_st * bits // 8), dtype=torch.uint8, device="cuda")
    w = qc.qconv_prepare_weights(d, torch.from_numpy(lp.w_bytes.reshape(-1).copy()).cuda()); d.w_prepared = 1
    m, n = qc.qconv_requant_params(lp.s_x, lp.s_w, lp.s_y)
    b = torch.from_numpy(lp.bias).cuda(); mm = torch.from_numpy(m).cuda(); nn = torch.from_numpy(n).cuda()
    for _ in range(2):
        y = qc.qconv2d_forward(d, x, w, b, mm, nn)
    torch.cuda.synchronize()
t = np.fromfile(out, dtype=np.uint64).reshape(-1, 16, 1024).astype(np.int64)[-1]
names = ["prod_empty_ok", "-", "mma_tempty_ok", "mma_full_ok", "mma_commit_tfull", "epi_tfull_ok", "epi_tempty_arrive", "epi_store_issued", "cvt_full_ok", "cvt_done", "cvt_loop_done"]
t0 = min(v for v in t.reshape(-1) if v > 0)
for ev, nm in enumerate(names):
    row = t[ev]
    row = row[row > 0] - t0
    if len(row):
        print(f"{nm:20s} n={len(row):4d} first={row[:6].tolist()} ... dt_avg={np.diff(row).mean() if len(row)>1 else 0:.0f} ns")
