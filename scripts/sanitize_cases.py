"""Small launches of every kernel family, for compute-sanitizer (memcheck / racecheck /
synccheck): halo (8- and 4-bit), channel-major, CTA pair (cluster), im2col (plain, x_zero /
w_zero, float output), the prep kernels, and two layers back to back on one stream (PDL).
Each result is compared with the oracle, so a run also shows the sanitizer left the bytes
unchanged.  Usage: python scripts/sanitize_cases.py"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc  # noqa: E402
from workloads import ConvShape, make_layer_inputs  # noqa: E402

DEV = "cuda:0"


def run(cs, bits, kernel, bn=0, x_zero=0, zw=False, dq=False, relu=True):
    li = make_layer_inputs(cs, bits, seed=cs.k + bits, relu=relu, x_zero=x_zero)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    wz = np.arange(cs.k, dtype=np.int32) % 5 - 2 if zw else None
    wz_d = None if wz is None else torch.from_numpy(wz).to(DEV)
    yt = qc.QC_F32_OUT if dq else li.y_t
    d = qc.make_desc(cs.n, cs.h, cs.w, cs.c, cs.k, cs.r, cs.s, stride=cs.stride, pad=cs.pad,
                     x_t=li.x_t, w_t=li.w_t, y_t=yt, x_zero=li.x_zero, clamp_lo=li.clamp_lo if not dq else 0,
                     clamp_hi=li.clamp_hi if not dq else 0, w_zero=wz_d)
    x = torch.from_numpy(li.x_bytes).to(DEV)
    w = torch.from_numpy(li.w_bytes).to(DEV)
    b = torch.from_numpy(li.bias).to(DEV)
    if kernel:
        qc.qconv_plan_set(d, kernel, bn)
    if dq:
        sc = (np.float32(li.s_x) * li.s_w).astype(np.float32)
        y = qc.qconv2d_forward_dequant(d, x, w, b, torch.from_numpy(sc).to(DEV))
        ref = oracle.conv2d_layer(li, y_t=oracle.F32, dq_scale=sc, w_zero=wz)
    else:
        y = qc.qconv2d_forward(d, x, w, b, torch.from_numpy(m).to(DEV), torch.from_numpy(n).to(DEV))
        ref = oracle.conv2d_layer(li, mult=m, shift=n, w_zero=wz)
    torch.cuda.synchronize()
    plan = qc.qconv_debug_plan(d)
    if kernel:
        qc.qconv_plan_set(d, None)
    got = y.cpu().numpy()
    ok = np.array_equal(got.view(np.uint8), ref.view(np.uint8))
    print(f"{cs.name:10s} {bits}-bit {plan['kernel_name']:8s} bn={plan['bn']:3d} "
          f"{'ok' if ok else 'MISMATCH'}", flush=True)
    return ok


def chain_pdl():
    """Two dependent layers enqueued back to back (the second reads the first's output): the
    programmatic-dependent-launch ordering."""
    cs1 = ConvShape("pdl1", 2, 14, 14, 64, 64, 3, 3, 1, 1)
    li = make_layer_inputs(cs1, 4, seed=1, relu=True)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    d = qc.make_desc(2, 14, 14, 64, 64, 3, 3, pad=1, x_t=li.x_t, w_t=li.w_t, y_t=li.y_t,
                     clamp_lo=li.clamp_lo, clamp_hi=li.clamp_hi)
    w = qc.qconv_prepare_weights(d, torch.from_numpy(li.w_bytes).to(DEV))
    d.w_prepared = 1
    b, mm, nn = (torch.from_numpy(a).to(DEV) for a in (li.bias, m, n))
    y1 = qc.qconv2d_forward(d, torch.from_numpy(li.x_bytes).to(DEV), w, b, mm, nn)
    y2 = qc.qconv2d_forward(d, y1, w, b, mm, nn)
    torch.cuda.synchronize()
    r1 = oracle.conv2d_layer(li, mult=m, shift=n)
    li.x_bytes = r1
    r2 = oracle.conv2d_layer(li, mult=m, shift=n)
    ok = np.array_equal(y2.cpu().numpy(), r2)
    print(f"pdl chain  4-bit {'ok' if ok else 'MISMATCH'}", flush=True)
    return ok


def fused_stem(bf16):
    """qconv2d_forward_quantize on a small C = 3 stem: the channel-major halo kernel quantizes
    the fp32 / bf16 rows itself (converter warps, code-row ring)."""
    from workloads import float_image, pack_codes, S8, U8
    cs = ConvShape("fstem", 1, 64, 64, 3, 64, 7, 7, 2, 3)
    rng = np.random.default_rng(9)
    xf = float_image(rng, (1, 64, 64, 3))
    s_x = 3.0 / 255
    li = make_layer_inputs(cs, 8, seed=11, c_store=4, relu=True)
    xt = torch.from_numpy(xf)
    if bf16:
        xt = xt.to(torch.bfloat16)
        host = xt.view(torch.int16).numpy().view(np.uint16)
    else:
        host = xf
    li.x_bytes = oracle.quantize(host, s_x, 0, U8, c_pad=4, bf16=bf16)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    d = qc.make_desc(1, 64, 64, 3, 64, 7, 7, stride=2, pad=3, x_t=U8, w_t=S8, y_t=li.y_t,
                     clamp_lo=li.clamp_lo, clamp_hi=li.clamp_hi)
    w = torch.from_numpy(np.ascontiguousarray(pack_codes(li.w_codes[..., :3], S8))).to(DEV)
    b, mm, nn = (torch.from_numpy(a).to(DEV) for a in (li.bias, m, n))
    y = qc.qconv2d_forward_quantize(d, xt.to(DEV).contiguous(), s_x, w, b, mm, nn)
    torch.cuda.synchronize()
    ok = np.array_equal(y.cpu().numpy(), ref)
    print(f"fused stem ({'bf16' if bf16 else 'fp32'}) {qc.qconv_debug_plan_quantize(d)['kernel_name']} "
          f"{'ok' if ok else 'MISMATCH'}", flush=True)
    return ok


def main():
    oks = [
        run(ConvShape("halot8", 2, 14, 14, 64, 64, 3, 3, 1, 1), 8, qc.QC_KERNEL_HALO_T),
        run(ConvShape("halot4", 2, 14, 14, 64, 64, 3, 3, 1, 1), 4, qc.QC_KERNEL_HALO_T),
        fused_stem(False),
        fused_stem(True),
        run(ConvShape("halo8", 2, 14, 14, 64, 64, 3, 3, 1, 1), 8, qc.QC_KERNEL_HALO),
        run(ConvShape("halo4", 2, 14, 14, 64, 64, 3, 3, 1, 1), 4, qc.QC_KERNEL_HALO),
        run(ConvShape("chan8", 2, 8, 16, 64, 128, 1, 1), 8, qc.QC_KERNEL_CHANNEL, 128),
        run(ConvShape("chan4", 2, 8, 16, 64, 64, 1, 1), 4, qc.QC_KERNEL_CHANNEL, 64),
        run(ConvShape("pair8", 2, 9, 9, 64, 128, 3, 3, 1, 1), 8, qc.QC_KERNEL_PAIR, 128),
        run(ConvShape("pair4", 2, 9, 9, 64, 128, 3, 3, 1, 1), 4, qc.QC_KERNEL_PAIR, 128),
        run(ConvShape("im2c8", 2, 9, 9, 64, 48, 3, 3, 2, 1), 8, qc.QC_KERNEL_IM2COL, 48),
        run(ConvShape("im2c4", 2, 9, 9, 64, 64, 3, 3, 2, 1), 4, qc.QC_KERNEL_IM2COL, 64),
        run(ConvShape("zxzw", 2, 9, 9, 64, 32, 3, 3, 1, 1), 8, 0, x_zero=20, zw=True),
        run(ConvShape("deq", 2, 9, 9, 64, 32, 3, 3, 1, 1), 4, 0, dq=True, relu=False),
        run(ConvShape("stem", 1, 32, 32, 3, 64, 7, 7, 2, 3), 8, 0),
        chain_pdl(),
    ]
    print("ALL OK" if all(oks) else "FAILURES")


if __name__ == "__main__":
    main()
