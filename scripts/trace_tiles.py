"""Debug builds only (-DQC_DEBUG): run one layer with QC_TRACE and print CTA 0's per-tile
pipeline timestamps (SM cycles) for the channel-major / im2col kernels.
usage: python scripts/trace_tiles.py layer:bits [layer:bits ...]"""
import os, sys, numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
out = "/tmp/qc_trace.bin"
os.environ["QC_TRACE"] = out
import torch
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc
import workloads as W
names = {0: "prod", 2: "mma_tempty", 3: "mma_full", 13: "mma_issued", 4: "mma_commit", 5: "epi_tfull",
         11: "epi_sfree", 6: "epi_done", 14: "epi1_tfull", 15: "epi1_done", 7: "store", 8: "cvt_full", 9: "cvt_arrive"}
for spec in sys.argv[1:]:
    name, bits = spec.split(':'); bits = int(bits)
    if os.path.exists(out): os.remove(out)
    cs = next(c for c in W.resnet50_convs(256) if c.name == name)
    c_st = W.stored_channels(cs, bits)
    lp = W.make_layer_params(cs, bits, 1, c_store=c_st)
    xt = W.U4 if bits == 4 else W.U8
    d = qc.make_desc(cs.n, cs.h, cs.w, c_st, cs.k, cs.r, cs.s, stride=cs.stride, pad=cs.pad, x_t=xt, w_t=lp.w_t, y_t=xt, relu=True)
    x = torch.randint(0, 255, (cs.n, cs.h, cs.w, c_st * bits // 8), dtype=torch.uint8, device="cuda")
    w = qc.qconv_prepare_weights(d, torch.from_numpy(lp.w_bytes.reshape(-1).copy()).cuda()); d.w_prepared = 1
    m, n = qc.qconv_requant_params(lp.s_x, lp.s_w, lp.s_y)
    b = torch.from_numpy(lp.bias).cuda(); mm = torch.from_numpy(m).cuda(); nn = torch.from_numpy(n).cuda()
    for _ in range(3):
        y = qc.qconv2d_forward(d, x, w, b, mm, nn)
    torch.cuda.synchronize()
    t = np.fromfile(out, dtype=np.uint64).reshape(-1, 16, 1024).astype(np.int64)[-1]
    t0 = min(v for v in t.reshape(-1) if v > 0)
    print(f"== {spec}  plan={qc.qconv_debug_plan(d) if hasattr(qc, 'qconv_debug_plan') else ''}")
    for ev, nm in names.items():
        row = t[ev]; row = row[row > 0] - t0
        if len(row):
            print(f"  {nm:11s} n={len(row):4d} " + " ".join(f"{v:7d}" for v in row[:14]))
    last = max(v for v in t.reshape(-1) if v > 0) - t0
    print(f"  CTA0 span {last} cycles")
