"""Round-2 ablations after the paper's Fig.11 and Fig.12, on the paper's 19 unique ResNet-50
layers at batch 1, L2 flushed before every timed launch, CUDA events:

Fig.11 (profile runs): per layer and bit width, the time with
  * fixed  -- one fixed tiling for every shape (the im2col kernel, N tile = min(K, 256)),
  * rule   -- the library's default kernel/tile rule,
  * tuned  -- the best candidate of qconv_autotune's profile runs.
Fig.12 (quantization fusion, P:L263-265, 8-bit, batch 1):
  * dequant fused   -- qconv2d_forward_dequant (fp32 straight from the epilogue)
    vs unfused      -- int32 output, then a separate elementwise dequantization (torch op)
  * ReLU fused      -- the truncation range lo = z_y in the requant epilogue
    vs unfused      -- full-range output, then a separate elementwise clamp (torch op)
Every variant's output is checked byte-for-byte against the fused one (same integer result).
Usage: python scripts/fig11_fig12.py out.json"""
import json
import os
import statistics
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc  # noqa: E402
import workloads as W  # noqa: E402

DEV = torch.device("cuda", 0)
FLUSH = torch.empty(512 << 20, dtype=torch.uint8, device=DEV)


def timeit(fn, steps=30, warm=5):
    for _ in range(warm):
        fn()
    ts = []
    for i in range(steps):
        FLUSH.fill_(i & 0xFF)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        ts.append((a, b))
    torch.cuda.synchronize()
    return statistics.median(a.elapsed_time(b) * 1e3 for a, b in ts)


def layer(cs, bits, seed):
    x_t, w_t = (W.U4, W.S4) if bits == 4 else (W.U8, W.S8)
    lp = W.make_layer_params(cs, bits, seed)
    d = qc.make_desc(cs.n, cs.h, cs.w, cs.c, cs.k, cs.r, cs.s, stride=cs.stride, pad=cs.pad,
                     x_t=x_t, w_t=w_t, y_t=x_t, relu=True)
    w = qc.qconv_prepare_weights(d, torch.from_numpy(np.ascontiguousarray(lp.w_bytes)).to(DEV))
    d.w_prepared = 1
    m, n = qc.qconv_requant_params(lp.s_x, lp.s_w, lp.s_y)
    x = W.device_post_relu_codes((cs.n, cs.h, cs.w, cs.c), bits, seed + 1, DEV)
    t = dict(d=d, w=w, b=torch.from_numpy(lp.bias).to(DEV), m=torch.from_numpy(m).to(DEV),
             n=torch.from_numpy(n).to(DEV), x=x, lp=lp)
    return t


def fig11(bits):
    rows = []
    for i, cs in enumerate(W.resnet50_unique(1)):
        L = layer(cs, bits, 500 + i)
        d = L["d"]
        y = qc.qconv2d_forward(d, L["x"], L["w"], L["b"], L["m"], L["n"])
        ref = y.clone()
        run = lambda: qc.qconv2d_forward(d, L["x"], L["w"], L["b"], L["m"], L["n"], y=y)
        qc.qconv_plan_set(d, None)
        rule = qc.qconv_debug_plan(d)
        t_rule = timeit(run)
        qc.qconv_plan_set(d, qc.QC_KERNEL_IM2COL, min(256, (cs.k + 15) // 16 * 16))
        t_fixed = timeit(run)
        assert torch.equal(y, ref)
        qc.qconv_plan_set(d, None)
        best, _ = qc.qconv_autotune(d, L["x"], L["w"], L["b"], L["m"], L["n"], y=y, iters=10)
        t_tuned = timeit(run)
        assert torch.equal(y, ref)
        qc.qconv_plan_set(d, None)
        rows.append({"layer": cs.name, "fixed_us": t_fixed, "rule_us": t_rule, "tuned_us": t_tuned,
                     "rule": f"{rule['kernel_name']}/{rule['bn']}",
                     "tuned": f"{best['kernel_name']}/{best['bn']}"})
    geo = lambda k: float(np.exp(np.mean([np.log(r["fixed_us"] / r[k]) for r in rows])))
    return {"bits": bits, "batch": 1, "layers": rows, "speedup_rule_vs_fixed_geomean": geo("rule_us"),
            "speedup_tuned_vs_fixed_geomean": geo("tuned_us")}


def fig12():
    rows = []
    for i, cs in enumerate(W.resnet50_unique(1)):
        L = layer(cs, 8, 700 + i)
        d = L["d"]
        lp = L["lp"]
        scale = torch.from_numpy((np.float32(lp.s_x) * lp.s_w).astype(np.float32)).to(DEV)
        # dequantization: fused fp32 epilogue vs int32 output + separate dequantize
        df = qc.qconv_desc.from_buffer_copy(d)
        df.y_t, df.clamp_lo, df.clamp_hi, df.relu = qc.QC_F32_OUT, 0, 0, 0
        di = qc.qconv_desc.from_buffer_copy(d)
        di.y_t, di.clamp_lo, di.clamp_hi = qc.QC_S32, 0, 0
        yf = qc.qconv2d_forward_dequant(df, L["x"], L["w"], L["b"], scale)
        yi = qc.qconv2d_forward(di, L["x"], L["w"], L["b"])
        fused_dq = lambda: qc.qconv2d_forward_dequant(df, L["x"], L["w"], L["b"], scale, y=yf)
        out = torch.empty_like(yf)

        def unfused_dq():
            qc.qconv2d_forward(di, L["x"], L["w"], L["b"], y=yi)
            torch.mul(yi.float(), scale, out=out)
        unfused_dq()
        torch.cuda.synchronize()
        assert torch.equal(out, yf), cs.name            # fl32(acc) * scale, RNE both ways
        # ReLU: truncation range in the epilogue vs full range + separate clamp
        dr = qc.qconv_desc.from_buffer_copy(d)
        dr.y_t, dr.clamp_lo, dr.clamp_hi = qc.QC_S8, 0, 127          # fused ReLU (z_y = 0)
        dn = qc.qconv_desc.from_buffer_copy(d)
        dn.y_t, dn.clamp_lo, dn.clamp_hi = qc.QC_S8, -128, 127
        yr = qc.qconv2d_forward(dr, L["x"], L["w"], L["b"], L["m"], L["n"])
        yn = qc.qconv2d_forward(dn, L["x"], L["w"], L["b"], L["m"], L["n"])
        fused_relu = lambda: qc.qconv2d_forward(dr, L["x"], L["w"], L["b"], L["m"], L["n"], y=yr)

        def unfused_relu():
            qc.qconv2d_forward(dn, L["x"], L["w"], L["b"], L["m"], L["n"], y=yn)
            yn.view(torch.int8).clamp_(min=0)
        unfused_relu()
        torch.cuda.synchronize()
        assert torch.equal(yn, yr), cs.name
        rows.append({"layer": cs.name, "dequant_fused_us": timeit(fused_dq),
                     "dequant_unfused_us": timeit(unfused_dq), "relu_fused_us": timeit(fused_relu),
                     "relu_unfused_us": timeit(unfused_relu)})
    g = lambda a, b: float(np.exp(np.mean([np.log(r[b] / r[a]) for r in rows])))
    return {"bits": 8, "batch": 1, "layers": rows,
            "dequant_fusion_speedup_geomean": g("dequant_fused_us", "dequant_unfused_us"),
            "relu_fusion_speedup_geomean": g("relu_fused_us", "relu_unfused_us"),
            "unfused_note": "the separate elementwise step is a torch op (dequant: int32->fp32 * scale; "
                            "ReLU: clamp of the int8 codes), as in the paper's unfused layer sequence"}


if __name__ == "__main__":
    out = {"fig11": [fig11(4), fig11(8)], "fig12": fig12()}
    for f in out["fig11"]:
        print(f"fig11 {f['bits']}-bit: rule/fixed {f['speedup_rule_vs_fixed_geomean']:.2f}x, "
              f"tuned/fixed {f['speedup_tuned_vs_fixed_geomean']:.2f}x")
    print(f"fig12: dequant fusion {out['fig12']['dequant_fusion_speedup_geomean']:.2f}x, "
          f"ReLU fusion {out['fig12']['relu_fusion_speedup_geomean']:.2f}x")
    with open(sys.argv[1] if len(sys.argv) > 1 else "fig11_fig12.json", "w") as f:
        json.dump(out, f, indent=1)
