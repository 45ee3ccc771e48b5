"""GPU parity for the round-2 paths, byte for byte against the CPU oracle (P:L273 exactness,
SURVEY 8(c) P11): every re-quantization mode on every kernel family with the full legal
multiplier / shift domain, the TFLite double rounding (reading Z15), the dequantized float
outputs (Z16), per-channel weight zero points (Z1), A8W4, channel counts the kernels
do not take directly (the C = 3 stems through qconv2d_forward), and every candidate plan of
the tile search -- all candidates must give the same bytes.
"""
import zlib

import numpy as np
import pytest

import oracle
from workloads import (C1, S4, S8, S32, U4, U8, ConvShape, DTYPE_RANGE, make_layer_inputs,
                       pack_codes, float_image, vgg16_convs)

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA GPU", allow_module_level=True)

import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc  # noqa: E402

DEV = "cuda:0"
F32, BF16 = oracle.F32, oracle.BF16


def _desc(li, y_t=None, lo=None, hi=None, **kw):
    cs = li.shape
    yt = li.y_t if y_t is None else y_t
    packed = yt in (U4, S4, U8, S8)
    if lo is None:
        lo, hi = (li.clamp_lo, li.clamp_hi) if (packed and yt == li.y_t) else (DTYPE_RANGE[yt] if packed else (0, 0))
    return qc.make_desc(cs.n, cs.h, cs.w, li.x_codes.shape[-1], cs.k, cs.r, cs.s, stride=cs.stride,
                        pad=cs.pad, dil=cs.dil, x_t=li.x_t, w_t=li.w_t, y_t=yt, x_zero=li.x_zero,
                        y_zero=li.y_zero, clamp_lo=lo, clamp_hi=hi, **kw)


def _gpu(li, m=None, n=None, y_t=None, kernel=None, bn=0, dq=None, lo=None, hi=None, w_zero=None,
         prepared=False, **kw):
    wz = None if w_zero is None else torch.from_numpy(np.asarray(w_zero, np.int32)).to(DEV)
    d = _desc(li, y_t, lo, hi, w_zero=wz, **kw)
    x = torch.from_numpy(np.ascontiguousarray(li.x_bytes)).to(DEV)
    w = torch.from_numpy(np.ascontiguousarray(li.w_bytes)).to(DEV)
    if prepared:
        w = qc.qconv_prepare_weights(d, w)
        d.w_prepared = 1
    b = torch.from_numpy(li.bias).to(DEV)
    if kernel is not None:
        qc.qconv_plan_set(d, kernel, bn)
    try:
        if dq is not None:
            y = qc.qconv2d_forward_dequant(d, x, w, b, torch.from_numpy(dq).to(DEV))
        else:
            mm = None if m is None else torch.from_numpy(np.asarray(m, np.int32)).to(DEV)
            nn = None if n is None else torch.from_numpy(np.asarray(n, np.int32)).to(DEV)
            y = qc.qconv2d_forward(d, x, w, b, mm, nn)
        torch.cuda.synchronize()
        plan = qc.qconv_debug_plan(d)
    finally:
        if kernel is not None:
            qc.qconv_plan_set(d, None)
    out = y.cpu()
    if out.dtype == torch.bfloat16:
        out = out.view(torch.int16)
    out = out.numpy()
    if out.dtype == np.int16:
        out = out.view(np.uint16)
    return out, plan


def _assert_same(got, ref, what=""):
    assert got.shape == ref.shape, (got.shape, ref.shape)
    if got.dtype == np.float32:
        got, ref = got.view(np.uint32), ref.view(np.uint32)
    if not np.array_equal(got, ref):
        bad = np.argwhere(got != ref)
        raise AssertionError(f"{what}: {bad.shape[0]} mismatches of {ref.size}; first {bad[:4].tolist()} "
                             f"got {got[tuple(bad[0])]} ref {ref[tuple(bad[0])]}")


# one shape per kernel family, with the family forced through the plan API
FAMILY_SHAPES = {
    "halo": (ConvShape("halo", 2, 14, 14, 64, 128, 3, 3, 1, 1), qc.QC_KERNEL_HALO, 0),
    "halo_t": (ConvShape("halo_t", 2, 14, 14, 64, 64, 3, 3, 1, 1), qc.QC_KERNEL_HALO_T, 0),
    "channel": (ConvShape("chan", 2, 10, 12, 64, 128, 1, 1), qc.QC_KERNEL_CHANNEL, 128),
    "pair": (ConvShape("pair", 2, 9, 9, 64, 128, 3, 3, 1, 1), qc.QC_KERNEL_PAIR, 128),
    "im2col": (ConvShape("im2col", 2, 11, 9, 64, 128, 3, 3, 2, 1), qc.QC_KERNEL_IM2COL, 128),
}


def _requant_domain(k, rng):
    """Per-channel (m, shift) over the whole legal domain, 32-column chunks chosen so every
    epilogue mode is reached: chunk 0 the old mid-mode hole (0 < m < 2^30, shift 20..32),
    chunk 1 negative multipliers with fast shifts, chunk 2 m = 0 mixed with normalised
    multipliers at mid shifts, chunk 3 extreme shifts 1..8 and 60..62."""
    m = np.zeros(k, np.int64)
    n = np.zeros(k, np.int64)
    c = np.arange(k) % 128
    sel = c < 32
    m[sel] = rng.integers(1, 1 << 30, sel.sum()); n[sel] = rng.integers(20, 33, sel.sum())
    sel = (c >= 32) & (c < 64)
    m[sel] = -rng.integers(1, 1 << 31, sel.sum()); n[sel] = rng.integers(33, 53, sel.sum())
    sel = (c >= 64) & (c < 96)
    m[sel] = rng.choice([0, 1 << 30, (1 << 31) - 1, -(1 << 30), -(1 << 31)], sel.sum())
    n[sel] = rng.integers(20, 51, sel.sum())
    sel = c >= 96
    m[sel] = rng.integers(-(1 << 31), 1 << 31, sel.sum())
    n[sel] = rng.choice([1, 2, 5, 8, 60, 61, 62], sel.sum())
    return m.astype(np.int32), n.astype(np.int32)


@pytest.mark.parametrize("family", list(FAMILY_SHAPES))
@pytest.mark.parametrize("bits,out", [(8, "s8"), (8, "u8"), (4, "u4"), (4, "s4")])
def test_requant_full_domain_every_kernel(family, bits, out):
    cs, kern, bn = FAMILY_SHAPES[family]
    li = make_layer_inputs(cs, bits, seed=zlib.crc32(f"{family}{bits}{out}".encode()) % 997,
                           relu=out.startswith("u"), signed_out=out.startswith("s"))
    rng = np.random.default_rng(zlib.crc32(family.encode()) + bits)
    m, n = _requant_domain(max(cs.k, 128), rng)
    if cs.k < 128:      # K = 64 (channel-major halo): every other channel keeps all four chunk kinds
        m, n = m[::128 // cs.k].copy(), n[::128 // cs.k].copy()
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    got, plan = _gpu(li, m, n, kernel=kern, bn=bn)
    assert plan["kernel"] == kern
    _assert_same(got, ref, f"{family} {bits}-bit {out}")


def test_requant_mid_hole_worked_example():
    """VERDICT r1 example: 8-bit, m = 2^20, shift 25, acc + b = 1000 -> 31 (the round-1 mid
    mode gave 1)."""
    cs = ConvShape("w", 1, 4, 4, 32, 64, 1, 1)
    li = make_layer_inputs(cs, 8, seed=1, relu=False, signed_out=True)
    li.x_codes[:] = 0
    li.x_bytes = pack_codes(li.x_codes, li.x_t)
    li.bias[:] = 1000
    m = np.full(64, 1 << 20, np.int32)
    n = np.full(64, 25, np.int32)
    for family in ("channel", "im2col"):
        kern = FAMILY_SHAPES[family][1]
        got, _ = _gpu(li, m, n, kernel=kern, bn=64)
        assert (got.view(np.int8) == 31).all(), family


@pytest.mark.parametrize("family", list(FAMILY_SHAPES))
@pytest.mark.parametrize("bits", [8, 4])
def test_tflite_rounding_every_kernel(family, bits):
    """TFLite rounding on every kernel that takes it (the channel-major kernels do not: their
    epilogue would spill registers; such layers then run on another kernel, by the default rule)."""
    cs, kern, bn = FAMILY_SHAPES[family]
    if family in ("channel", "halo_t"):
        kern, bn = None, 0
    li = make_layer_inputs(cs, bits, seed=5 + bits, relu=False, signed_out=True)
    rng = np.random.default_rng(7 + bits)
    m, n = _requant_domain(cs.k, rng)
    ref = oracle.conv2d_layer(li, mult=m, shift=n, rounding=oracle.ROUND_TFLITE)
    got, _ = _gpu(li, m, n, kernel=kern, bn=bn, rounding=qc.QC_ROUND_TFLITE)
    _assert_same(got, ref, f"tflite {family} {bits}")
    mr, nr = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=mr, shift=nr, rounding=oracle.ROUND_TFLITE)
    got, _ = _gpu(li, mr, nr, kernel=kern, bn=bn, rounding=qc.QC_ROUND_TFLITE)
    _assert_same(got, ref, f"tflite R1 params {family} {bits}")


@pytest.mark.parametrize("cs", [ConvShape("d1", 2, 9, 11, 64, 48, 3, 3, 1, 1),
                                ConvShape("d2", 1, 14, 14, 128, 200, 1, 1, 2, 0),
                                ConvShape("d3", 3, 8, 8, 32, 16, 5, 5, 1, 2)], ids=lambda c: c.name)
@pytest.mark.parametrize("bits", [8, 4])
@pytest.mark.parametrize("yt", [F32, BF16])
@pytest.mark.parametrize("relu", [False, True])
def test_dequant_outputs(cs, bits, yt, relu):
    """Fusion of convolution and dequantization: fp32/bf16 straight from the
    epilogue; bias values at the fp32 rounding boundary included."""
    li = make_layer_inputs(cs, bits, seed=cs.k + bits, relu=False, signed_out=True)
    li.bias[:3] = [2 ** 24 + 1, -(2 ** 24 + 3), 2 ** 25 + 3]
    dq = (np.float32(li.s_x) * li.s_w).astype(np.float32)
    ref = oracle.conv2d_layer(li, y_t=yt, dq_scale=dq, relu=relu)
    got, plan = _gpu(li, y_t=qc.QC_F32_OUT if yt == F32 else qc.QC_BF16_OUT, dq=dq, relu=relu)
    assert plan["kernel_name"] == "im2col"
    _assert_same(got, ref, "dequant")


@pytest.mark.parametrize("bits", [8, 4])
def test_dequant_with_zero_points(bits):
    cs = ConvShape("dz", 2, 9, 9, 64, 40, 3, 3, 1, 1)
    li = make_layer_inputs(cs, bits, seed=3, x_zero=5 if bits == 4 else 90, relu=False, signed_out=True)
    dq = (np.float32(li.s_x) * li.s_w).astype(np.float32)
    zw = np.random.default_rng(4).integers(-3, 4, cs.k).astype(np.int32)
    ref = oracle.conv2d_layer(li, y_t=F32, dq_scale=dq, w_zero=zw)
    got, _ = _gpu(li, y_t=qc.QC_F32_OUT, dq=dq, w_zero=zw)
    _assert_same(got, ref, "dequant zx zw")


@pytest.mark.parametrize("cs", [ConvShape("z1", 2, 9, 11, 64, 48, 3, 3, 1, 1),
                                ConvShape("z2", 3, 10, 7, 32, 40, 3, 3, 2, 1),
                                ConvShape("z3", 1, 12, 12, 64, 64, 1, 1, 1, 0),
                                ConvShape("z4", 1, 12, 12, 32, 16, 3, 3, 1, 2, 2)], ids=lambda c: c.name)
@pytest.mark.parametrize("bits", [8, 4])
@pytest.mark.parametrize("x_zero", [0, 1])
def test_weight_zero_points(cs, bits, x_zero):
    """Per-output-channel weight zero points z_w[k] (reading Z1): the epilogue
    subtracts z_w[k] * sum over in-bounds taps of (x - x_zero)."""
    li = make_layer_inputs(cs, bits, seed=cs.k * 3 + bits, relu=True,
                           x_zero=(0 if not x_zero else (6 if bits == 4 else 77)))
    rng = np.random.default_rng(cs.k)
    lo, hi = DTYPE_RANGE[li.w_t]
    zw = rng.integers(lo // 2, hi // 2 + 1, cs.k).astype(np.int32)
    zw[:2] = [lo, hi]
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n, w_zero=zw)
    got, plan = _gpu(li, m, n, w_zero=zw)
    assert plan["prologue"] & 8
    _assert_same(got, ref, "w_zero")
    ref = oracle.conv2d_layer(li, y_t=S32, w_zero=zw)
    got, _ = _gpu(li, y_t=qc.QC_S32, w_zero=zw, lo=0, hi=0)
    _assert_same(got, ref, "w_zero s32")


def test_unsigned_weights_with_zero_point():
    """Asymmetric unsigned 8-bit weights (z_w = 128), the TFLite uint8 convention."""
    cs = ConvShape("uw", 2, 10, 10, 64, 64, 3, 3, 1, 1)
    li = make_layer_inputs(cs, 8, seed=8, relu=True)
    li.w_t = U8
    li.w_codes = np.clip(li.w_codes + 128, 0, 255)
    li.w_bytes = pack_codes(li.w_codes, U8)
    zw = np.full(cs.k, 128, np.int32)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n, w_zero=zw)
    got, _ = _gpu(li, m, n, w_zero=zw)
    _assert_same(got, ref, "u8 weights")


@pytest.mark.parametrize("cs", [ConvShape("a1", 2, 12, 12, 64, 64, 3, 3, 1, 1),
                                ConvShape("a2", 2, 14, 14, 128, 256, 1, 1, 1, 0),
                                ConvShape("a3", 1, 15, 15, 64, 96, 3, 3, 2, 1)], ids=lambda c: c.name)
@pytest.mark.parametrize("wt", [S4, U4])
def test_a8w4(cs, wt):
    """8-bit activations with 4-bit weights: weights widened once to int8."""
    li = make_layer_inputs(cs, 8, seed=cs.c + wt, relu=True)
    lo, hi = DTYPE_RANGE[wt]
    li.w_t = wt
    li.w_codes = np.random.default_rng(cs.k).integers(lo, hi + 1, li.w_codes.shape)
    li.w_bytes = pack_codes(li.w_codes, wt)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    got, _ = _gpu(li, m, n)
    _assert_same(got, ref, "A8W4")
    got, _ = _gpu(li, m, n, prepared=True)
    _assert_same(got, ref, "A8W4 prepared")


@pytest.mark.parametrize("bits", [8, 4])
@pytest.mark.parametrize("n_img,x_zero", [(2, 0), (1, 3)])
@pytest.mark.parametrize("prepared", [False, True])
def test_stem_c3_through_forward(bits, n_img, x_zero, prepared):
    """The 7x7/s2/p3 stem with its true channel count through qconv2d_forward (space-to-depth
    chosen inside the library; 4-bit rows need an even count, so C = 4 with a zero-point
    channel)."""
    from workloads import resnet50_convs
    base = resnet50_convs(n_img)[0]
    c = 3 if bits == 8 else 4
    cs = ConvShape("stem", n_img, 224, 224, c, 64, 7, 7, 2, 3)
    li = make_layer_inputs(cs, bits, seed=11 + bits, x_zero=x_zero)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    got, plan = _gpu(li, m, n, prepared=prepared)
    assert plan["prologue"] & 2
    assert base.k == cs.k
    _assert_same(got, ref, "stem")


@pytest.mark.parametrize("cs,bits", [
    (ConvShape("vgg1_1", 2, 32, 32, 3, 64, 3, 3, 1, 1), 8),
    (ConvShape("c48", 2, 9, 9, 48, 64, 3, 3, 1, 1), 8),
    (ConvShape("c20_4", 2, 9, 9, 20, 32, 3, 3, 2, 1), 4),
    (ConvShape("c8", 1, 10, 10, 8, 32, 1, 1, 1, 0), 8),
    (ConvShape("c6_4", 1, 11, 13, 6, 64, 5, 5, 1, 2), 4),
], ids=lambda v: getattr(v, "name", str(v)))
def test_channel_padding(cs, bits):
    li = make_layer_inputs(cs, bits, seed=cs.c * 7 + bits, relu=True)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    got, plan = _gpu(li, m, n)
    assert plan["prologue"] & 2
    _assert_same(got, ref, cs.name)


def test_vgg16_conv1_1_batch2():
    """VGG-16 conv1_1 (C = 3, 3x3/s1, 224x224), the layer round 1 could not run.  Its codes are
    padded to 16 channels and its filter to 3x4 (a zero-weight column, one zero-point input
    column) so the channel-major halo kernel pairs its taps -- checked to be the plan taken."""
    cs = vgg16_convs(2)[0]
    li = make_layer_inputs(cs, 8, seed=3000)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    got, plan = _gpu(li, m, n)
    assert plan["kernel_name"] == "halo_t", plan
    _assert_same(got, ref, "vgg conv1_1")


@pytest.mark.parametrize("cs", [
    ConvShape("c3s5", 2, 20, 23, 3, 32, 5, 5, 1, 2),        # odd S = 5 -> 6, pixel-major halo
    ConvShape("c7s3", 3, 16, 29, 7, 64, 3, 3, 1, 1),        # K = 64 -> channel-major halo
    ConvShape("c1s1x3", 2, 12, 40, 1, 64, 1, 3, 1, 0),      # 1x3 filter, no padding
], ids=lambda v: v.name)
def test_odd_filter_width_tap_pairs(cs):
    """8-bit, C < 16, stride 1, odd S: the filter gains a zero-weight column and the input a
    zero-point column (same products, same P x Q) so a halo kernel can pair taps."""
    li = make_layer_inputs(cs, 8, seed=cs.c * 13 + cs.s, relu=True)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    for prepared in (False, True):
        got, plan = _gpu(li, m, n, prepared=prepared)
        assert plan["kernel_name"] in ("halo", "halo_t"), plan
        _assert_same(got, ref, f"{cs.name} prepared={prepared}")


TUNE_SHAPES = [ConvShape("t3", 4, 14, 14, 128, 128, 3, 3, 1, 1),
               ConvShape("t1", 4, 14, 14, 256, 128, 1, 1, 1, 0),
               ConvShape("t1s", 4, 28, 28, 256, 512, 1, 1, 2, 0),
               ConvShape("t7", 2, 28, 28, 64, 64, 3, 3, 1, 1)]


@pytest.mark.parametrize("cs", TUNE_SHAPES, ids=lambda c: c.name)
@pytest.mark.parametrize("bits", [8, 4])
def test_every_candidate_plan_is_exact(cs, bits):
    """The tile search may pick any candidate: each gives the oracle's bytes."""
    li = make_layer_inputs(cs, bits, seed=cs.k + cs.r + bits, relu=True)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    d = _desc(li)
    cands = qc.qconv_plan_candidates(d)
    assert len(cands) >= 3
    for c in cands:
        got, plan = _gpu(li, m, n, kernel=c["kernel"], bn=c["bn"])
        assert (plan["kernel"], plan["bn"]) == (c["kernel"], c["bn"])
        _assert_same(got, ref, f"{cs.name} {c['kernel_name']} bn={c['bn']}")


def test_autotune_records_an_exact_plan():
    cs = TUNE_SHAPES[0]
    li = make_layer_inputs(cs, 4, seed=21, relu=True)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    d = _desc(li)
    x = torch.from_numpy(li.x_bytes).to(DEV)
    w = torch.from_numpy(li.w_bytes).to(DEV)
    b = torch.from_numpy(li.bias).to(DEV)
    mm, nn = torch.from_numpy(m).to(DEV), torch.from_numpy(n).to(DEV)
    best, us = qc.qconv_autotune(d, x, w, b, mm, nn, iters=3)
    assert us > 0 and qc.qconv_debug_plan(d)["kernel"] == best["kernel"]
    y = qc.qconv2d_forward(d, x, w, b, mm, nn)
    torch.cuda.synchronize()
    _assert_same(y.cpu().numpy(), ref, "autotuned")
    qc.qconv_plan_set(d, None)


@pytest.mark.parametrize("bits", [8, 4])
@pytest.mark.parametrize("n_img,relu,bf16", [(2, True, False), (1, False, False), (5, True, False),
                                             (2, True, True), (3, False, True)])
@pytest.mark.parametrize("kernel", ["halo_t", "halo"])
def test_forward_quantize_fused_stem(bits, n_img, relu, bf16, kernel):
    """qconv2d_forward_quantize on the C = 3 stem: one kernel quantizes the fp32 (or bf16) rows
    (Z4) into its space-to-depth operand tile; compared with oracle quantize (+ a zero-point
    channel) then the oracle's direct 7x7/s2 conv.  Inputs include NaN, +-inf and exact
    quantization ties (in bf16: the bf16 roundings of them)."""
    cs = ConvShape("stem", n_img, 224, 224, 3, 64, 7, 7, 2, 3)
    rng = np.random.default_rng(60 + bits + n_img)
    xf = float_image(rng, (n_img, 224, 224, 3))
    s_x = 3.0 / 15 if bits == 4 else 3.0 / 255
    xf.reshape(-1)[:6] = [np.nan, np.inf, -np.inf, 0.5 * s_x, 1.5 * s_x, 2.5 * s_x]
    xt = U4 if bits == 4 else U8
    li = make_layer_inputs(cs, bits, seed=3 + bits, c_store=4, relu=relu, signed_out=not relu)
    xtensor = torch.from_numpy(xf)
    if bf16:
        xtensor = xtensor.to(torch.bfloat16)
        host = xtensor.view(torch.int16).numpy().view(np.uint16)
    else:
        host = xf
    li.x_bytes = oracle.quantize(host, s_x, 0, xt, c_pad=4, bf16=bf16)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    d = qc.make_desc(n_img, 224, 224, 3, 64, 7, 7, stride=2, pad=3, x_t=xt, w_t=S8, y_t=li.y_t,
                     clamp_lo=li.clamp_lo, clamp_hi=li.clamp_hi)
    w = torch.from_numpy(np.ascontiguousarray(pack_codes(li.w_codes[..., :3], S8))).to(DEV)
    b, mm, nn = (torch.from_numpy(a).to(DEV) for a in (li.bias, m, n))
    want = qc.QC_KERNEL_HALO_T if kernel == "halo_t" else qc.QC_KERNEL_HALO
    try:
        for prepared in (False, True):
            if prepared:
                w = qc.qconv_prepare_weights(d, w)
                d.w_prepared = 1
                assert qc._lib().qconv2d_quantize_workspace_size(d, qc.QC_BF16 if bf16 else qc.QC_F32) == 0   # one kernel
            if kernel == "halo":        # the pixel-major halo, chosen through the plan API
                qc.qconv_plan_set(d, qc.QC_KERNEL_HALO, 0)
            assert qc.qconv_debug_plan_quantize(d)["kernel"] == want
            y = qc.qconv2d_forward_quantize(d, xtensor.to(DEV).contiguous(), s_x, w, b, mm, nn)
            torch.cuda.synchronize()
            _assert_same(y.cpu().numpy(), ref, f"fused stem {kernel} (prepared={prepared}, bf16={bf16})")
    finally:
        qc.qconv_plan_clear()


@pytest.mark.parametrize("cs,bits,x_zero,bf16", [
    (ConvShape("q1", 2, 9, 11, 64, 48, 3, 3, 1, 1), 8, 0, False),
    (ConvShape("q2", 2, 12, 12, 32, 64, 1, 1), 4, 3, True),
    (ConvShape("q3", 1, 32, 32, 3, 16, 7, 7, 2, 3), 8, 5, False),      # stem shape, x_zero: two launches
], ids=lambda v: getattr(v, "name", str(v)))
def test_forward_quantize_general(cs, bits, x_zero, bf16):
    """Descriptors outside the fused stem case: quantize into the workspace, then the conv."""
    rng = np.random.default_rng(cs.c + bits)
    xf = rng.normal(0.5, 1.0, size=(cs.n, cs.h, cs.w, cs.c)).astype(np.float32)
    xt = U4 if bits == 4 else U8
    s_x = 0.11
    xtensor = torch.from_numpy(xf)
    if bf16:
        xtensor = xtensor.to(torch.bfloat16)
        host = xtensor.view(torch.int16).numpy().view(np.uint16)
    else:
        host = xf
    li = make_layer_inputs(cs, bits, seed=cs.k, relu=True, x_zero=x_zero)
    li.x_bytes = oracle.quantize(host, s_x, x_zero, xt, bf16=bf16)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    d = _desc(li)
    b, mm, nn = (torch.from_numpy(a).to(DEV) for a in (li.bias, m, n))
    y = qc.qconv2d_forward_quantize(d, xtensor.to(DEV).contiguous(), s_x,
                                    torch.from_numpy(li.w_bytes).to(DEV), b, mm, nn)
    torch.cuda.synchronize()
    _assert_same(y.cpu().numpy(), ref, cs.name)
