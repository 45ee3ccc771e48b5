"""Per-tile pipeline timeline (SM clock cycles) of CTA 0 for one layer (QC_DEBUG build, QC_TRACE): the MMA
warp's accumulator waits and commits, the epilogue's accumulator / staging waits and finish,
the storer's issues.  Usage: python scripts/trace_timeline.py out.bin res2a_branch2c:4"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
out = sys.argv[1]
os.environ["QC_TRACE"] = out
if os.path.exists(out):
    os.remove(out)
import torch  # noqa: E402
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc  # noqa: E402
import workloads as W  # noqa: E402

name, bits = sys.argv[2].split(":")
bits = int(bits)
cs = next(c for c in W.resnet50_convs(256) if c.name == name)
c_st = W.stored_channels(cs, bits)
lp = W.make_layer_params(cs, bits, 1, c_store=c_st)
xt = W.U4 if bits == 4 else W.U8
d = qc.make_desc(cs.n, cs.h, cs.w, c_st, cs.k, cs.r, cs.s, stride=cs.stride, pad=cs.pad, x_t=xt,
                 w_t=lp.w_t, y_t=xt, relu=True)
x = W.device_post_relu_codes((cs.n, cs.h, cs.w, c_st), bits, 1, "cuda")
w = qc.qconv_prepare_weights(d, torch.from_numpy(lp.w_bytes.reshape(-1).copy()).cuda())
d.w_prepared = 1
m, n = qc.qconv_requant_params(lp.s_x, lp.s_w, lp.s_y)
b, mm, nn = (torch.from_numpy(a).cuda() for a in (lp.bias, m, n))
print(qc.qconv_debug_plan(d))
for _ in range(3):
    qc.qconv2d_forward(d, x, w, b, mm, nn)
torch.cuda.synchronize()
t = np.fromfile(out, dtype=np.uint64).reshape(-1, 16, 1024).astype(np.int64)[-1]
t0 = min(v for v in t.reshape(-1) if v > 0)
cols = [(2, "mma_acc_free"), (4, "mma_commit"), (5, "epi_acc_full"), (1, "epi_stg_free"),
        (6, "epi_done"), (7, "store_issued")]
print("tile " + " ".join(f"{nm:>13s}" for _, nm in cols))
ntiles = int((t[5] > 0).sum())
for it in list(range(min(ntiles, 12))) + list(range(max(12, ntiles - 4), ntiles)):
    print(f"{it:4d} " + " ".join(f"{(t[ev, it] - t0) if t[ev, it] > 0 else -1:13d}" for ev, _ in cols))
epi = t[6, :ntiles] - t[5, :ntiles]
gap = t[5, 1:ntiles] - t[6, :ntiles - 1]
print(f"tiles {ntiles}; epilogue busy per tile {epi.mean():.0f} cyc; waiting for the accumulator "
      f"between tiles {gap.mean():.0f} cyc; total {(t[6, ntiles - 1] - t[5, 0]) / 1965:.1f} us")
for ev, nm in [(14, "prod_top"), (0, "producer"), (13, "prod_issued"), (3, "mma_stage_in"), (11, "mma_issued"), (12, "cvt_full_ok"), (8, "cvt_in"), (9, "cvt_done")]:
    row = t[ev][t[ev] > 0] - t0
    if len(row) > 1:
        print(f"{nm:14s} n={len(row)} first {row[:10].tolist()} mean dt {np.diff(row).mean():.0f} cyc")
