"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, byte for byte.

The paper claims its kernels "guarantee the same results as 32-bit computation"
(P:L273); every comparison below is therefore exact equality of the packed
output bytes (pin P11).  Inputs come from workloads/ (seeded);
requant parameters fed to both sides come from the oracle.
"""
import zlib

import numpy as np
import pytest

import oracle
from workloads import (C1, S4, S8, S32, U4, U8, ConvShape, DTYPE_RANGE, make_layer_inputs,
                       pack_codes, resnet50_convs, stored_channels, float_image, unpack_codes,
                       vgg16_convs)

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA GPU", allow_module_level=True)

import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc  # noqa: E402

DEV = "cuda:0"


def _desc_for(li, y_t=None, w_prepared=0):
    cs = li.shape
    c_st = li.x_codes.shape[-1]
    yt = li.y_t if y_t is None else y_t
    lo, hi = (li.clamp_lo, li.clamp_hi) if yt == li.y_t else (None, None)
    return qc.make_desc(cs.n, cs.h, cs.w, c_st, cs.k, cs.r, cs.s, stride=cs.stride, pad=cs.pad,
                        dil=cs.dil, x_t=li.x_t, w_t=li.w_t, y_t=yt, x_zero=li.x_zero,
                        y_zero=li.y_zero, clamp_lo=lo if yt != S32 else 0,
                        clamp_hi=hi if yt != S32 else 0, w_prepared=w_prepared)


def _gpu_conv(li, m, n, y_t=None, bias=True, prepared=False):
    d = _desc_for(li, y_t)
    x = torch.from_numpy(li.x_bytes).to(DEV)
    w = torch.from_numpy(li.w_bytes).to(DEV)
    if prepared:
        w = qc.qconv_prepare_weights(d, w)
        d.w_prepared = 1
    b = torch.from_numpy(li.bias).to(DEV) if bias else None
    mm = None if m is None else torch.from_numpy(m).to(DEV)
    nn = None if n is None else torch.from_numpy(n).to(DEV)
    y = qc.qconv2d_forward(d, x, w, b, mm, nn)
    torch.cuda.synchronize()
    return y.cpu().numpy()


def _check_layer(li, y_t=None, bias=True, prepared=False):
    yt = li.y_t if y_t is None else y_t
    if yt == S32:
        m = n = None
    else:
        m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n, y_t=yt, bias=bias)
    got = _gpu_conv(li, m, n, y_t=yt, bias=bias, prepared=prepared)
    assert got.shape == ref.shape
    if not np.array_equal(got, ref):
        bad = np.argwhere(got != ref)
        raise AssertionError(f"{bad.shape[0]} mismatching bytes of {ref.size}; first {bad[:5]} "
                             f"got {got[tuple(bad[0])]} ref {ref[tuple(bad[0])]}")
    return ref


# ----------------------------------------------------------------------------- TMA im2col
@pytest.mark.parametrize("cs,bits", [
    (ConvShape("a", 2, 9, 11, 32, 8, 3, 3, 1, 1), 8),
    (ConvShape("b", 3, 10, 7, 64, 8, 3, 3, 2, 1), 8),
    (ConvShape("c", 1, 12, 12, 32, 8, 3, 3, 1, 2, 2), 8),
    (ConvShape("d", 2, 14, 14, 64, 8, 1, 1, 2, 0), 8),
    (ConvShape("e", 2, 9, 9, 64, 8, 3, 3, 1, 1), 4),
    (ConvShape("f", 1, 23, 23, 32, 8, 7, 7, 2, 3), 8),
])
def test_im2col_tile_semantics(cs, bits):
    rng = np.random.default_rng(0)
    cbytes = cs.c * bits // 8
    xb = rng.integers(0, 256, size=(cs.n, cs.h, cs.w, cbytes), dtype=np.uint8)
    d = qc.make_desc(cs.n, cs.h, cs.w, cs.c, cs.k, cs.r, cs.s, stride=cs.stride, pad=cs.pad,
                     dil=cs.dil, x_t=U4 if bits == 4 else U8, w_t=S4 if bits == 4 else S8)
    x = torch.from_numpy(xb).to(DEV)
    M = cs.n * cs.p * cs.q
    box = 16 if cbytes == 16 else 32
    for m0 in sorted({0, 5, min(M - 1, 37), M - 1, M // 2}):
        for (r, s) in [(0, 0), (cs.r - 1, cs.s - 1), (cs.r // 2, 0)]:
            for cb in (0, cbytes - box):
                got = qc.qconv_debug_im2col_tile(d, x, m0, r, s, cb, box).cpu().numpy()
                exp = np.zeros((128, box), dtype=np.uint8)
                for i in range(128):
                    m = m0 + i
                    img, rem = divmod(m, cs.p * cs.q)
                    p, q = divmod(rem, cs.q)
                    hh = p * cs.stride - cs.pad + r * cs.dil
                    ww = q * cs.stride - cs.pad + s * cs.dil
                    if img < cs.n and 0 <= hh < cs.h and 0 <= ww < cs.w:
                        exp[i] = xb[img, hh, ww, cb:cb + box]
                np.testing.assert_array_equal(got, exp, err_msg=f"m0={m0} r={r} s={s} cb={cb}")


# ----------------------------------------------------------------------------- quantize_pack
@pytest.mark.parametrize("yt,zp", [(U8, 0), (S8, -3), (U4, 2), (S4, 0)])
@pytest.mark.parametrize("bf16", [False, True])
@pytest.mark.parametrize("c,c_pad", [(64, 64), (3, 32), (32, 48), (5, 6)])
def test_quantize_pack_parity(yt, zp, bf16, c, c_pad):
    rng = np.random.default_rng(c * 7 + c_pad)
    x = rng.normal(0, 2.0, size=(2, 7, 9, c)).astype(np.float32)
    x.reshape(-1)[:8] = [np.nan, np.inf, -np.inf, 0.5 * 0.13, 1.5 * 0.13, -2.5 * 0.13, 1e9, -0.0]
    xt = torch.from_numpy(x)
    if bf16:
        xt = xt.to(torch.bfloat16)
        host = xt.view(torch.int16).numpy().view(np.uint16)
    else:
        host = x
    got = qc.qconv_quantize_pack(xt.to(DEV).contiguous(), 0.13, zp, yt, c_pad=c_pad).cpu().numpy()
    ref = oracle.quantize(host, 0.13, zp, yt, c_pad=c_pad, bf16=bf16)
    np.testing.assert_array_equal(got, ref)


def test_quantize_pack_large_vector_path():
    rng = np.random.default_rng(3)
    x = rng.normal(0, 1, size=(4, 56, 56, 64)).astype(np.float32)
    got = qc.qconv_quantize_pack(torch.from_numpy(x).to(DEV), 3.0 / 15, 0, U4).cpu().numpy()
    np.testing.assert_array_equal(got, oracle.quantize(x, 3.0 / 15, 0, U4))


# ----------------------------------------------------------------------------- conv parity
SMALL_SHAPES = [
    ConvShape("s1", 1, 8, 8, 32, 16, 1, 1, 1, 0),
    ConvShape("s2", 2, 9, 11, 32, 48, 3, 3, 1, 1),
    ConvShape("s3", 3, 10, 7, 64, 40, 3, 3, 2, 1),
    ConvShape("s4", 1, 12, 12, 96, 32, 3, 3, 1, 2, 2),
    ConvShape("s5", 2, 14, 14, 128, 80, 1, 1, 2, 0),
    ConvShape("s6", 1, 17, 13, 256, 272, 3, 3, 1, 1),
    ConvShape("s7", 5, 6, 6, 64, 16, 5, 5, 1, 2),
    ConvShape("s8", 1, 30, 30, 32, 64, 7, 7, 2, 3),
]


@pytest.mark.parametrize("cs", SMALL_SHAPES, ids=lambda c: c.name)
@pytest.mark.parametrize("bits", [8, 4])
@pytest.mark.parametrize("out", ["same", "signed", "s32"])
def test_conv_small_shapes(cs, bits, out):
    li = make_layer_inputs(cs, bits, seed=zlib.crc32(f"{cs.name}{bits}{out}".encode()) % 1000,
                           signed_out=(out == "signed"), relu=(out == "same"),
                           out_bits=32 if out == "s32" else None)
    _check_layer(li)


@pytest.mark.parametrize("bits", [8, 4])
def test_conv_signed_activations_and_extremes(bits):
    cs = ConvShape("ext", 2, 9, 9, 64, 48, 3, 3, 1, 1)
    rng = np.random.default_rng(11)
    li = make_layer_inputs(cs, bits, seed=5, relu=False, signed_out=True)
    xt = S4 if bits == 4 else S8
    lo, hi = DTYPE_RANGE[xt]
    li.x_t = xt
    li.x_codes = rng.integers(lo, hi + 1, size=li.x_codes.shape)
    li.x_codes[0, :3] = lo
    li.x_codes[1, :3] = hi
    li.w_codes[:4] = DTYPE_RANGE[li.w_t][0]
    li.x_bytes = pack_codes(li.x_codes, xt)
    li.w_bytes = pack_codes(li.w_codes, li.w_t)
    _check_layer(li)
    _check_layer(li, y_t=S32)


@pytest.mark.parametrize("bits", [8, 4])
@pytest.mark.parametrize("pad", [0, 1])
def test_conv_x_zero_point(bits, pad):
    cs = ConvShape("zx", 2, 11, 9, 64, 32, 3, 3, 1, pad)
    li = make_layer_inputs(cs, bits, seed=17, x_zero=(7 if bits == 4 else 100), relu=True)
    _check_layer(li)
    _check_layer(li, y_t=S32)


def test_conv_no_bias_prepared_and_relu6_clamp():
    cs = ConvShape("nb", 1, 12, 12, 64, 64, 3, 3, 1, 1)
    li = make_layer_inputs(cs, 4, seed=2)
    _check_layer(li, bias=False, prepared=True)
    li.clamp_lo, li.clamp_hi = 1, 6          # ReLU6-style truncation range
    _check_layer(li, prepared=True)


def test_conv_requant_shift_modes():
    """Shifts below 32 and above 52 take the 64-bit epilogue branch."""
    cs = ConvShape("sh", 1, 8, 8, 32, 32, 1, 1, 1, 0)
    li = make_layer_inputs(cs, 8, seed=4, relu=False, signed_out=True)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    n = n.copy()
    m = m.copy()
    n[:8] = np.arange(20, 28)          # large multipliers (M > 1)
    n[8:16] = np.arange(53, 61)        # tiny multipliers
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    got = _gpu_conv(li, m, n)
    np.testing.assert_array_equal(got, ref)


@pytest.mark.parametrize("bits,lo_n,hi_n", [(8, 14, 33), (4, 14, 33), (8, 33, 52), (4, 28, 36)])
def test_conv_requant_shift_ranges(bits, lo_n, hi_n):
    """Random per-channel (m, shift) over whole 32-channel chunks: exercises the mid (shift
    14..33, pre-clamped and rescaled), fast (33..52) and mixed/general epilogue branches,
    including saturation, against the oracle's exact int128 rounding."""
    cs = ConvShape("shr", 2, 9, 9, 64, 96, 3, 3, 1, 1)
    li = make_layer_inputs(cs, bits, seed=lo_n * 7 + bits, relu=False, signed_out=True)
    rng = np.random.default_rng(lo_n + hi_n)
    m = rng.integers(1 << 30, 1 << 31, size=cs.k).astype(np.int32)
    n = rng.integers(lo_n, hi_n + 1, size=cs.k).astype(np.int32)
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    got = _gpu_conv(li, m, n)
    np.testing.assert_array_equal(got, ref)


# ----------------------------------------------------------------------------- paper configs
def test_config1_c1_8bit():
    """BASELINE configs[0]: 8-bit 3x3, N=1, C=K=64, 56x56, s1 p1, requantized int8 output."""
    _check_layer(make_layer_inputs(C1, 8, seed=20200817))
    _check_layer(make_layer_inputs(C1, 8, seed=20200818, uniform_x=True))


def test_config2_c2_4bit_with_quantize():
    """BASELINE configs[1]: same layer at A4W4, fp32 input -> quantize_pack -> conv -> u4 out."""
    rng = np.random.default_rng(20200817)
    xf = float_image(rng, (1, 56, 56, 64))
    li = make_layer_inputs(C1, 4, seed=20200817)
    s_x = 3.0 / 15
    xq_ref = oracle.quantize(xf, s_x, 0, U4)
    xq = qc.qconv_quantize_pack(torch.from_numpy(xf).to(DEV), s_x, 0, U4)
    np.testing.assert_array_equal(xq.cpu().numpy(), xq_ref)
    li.x_bytes = xq_ref
    li.x_codes = unpack_codes(xq_ref, U4, 64)
    _check_layer(li)


@pytest.mark.parametrize("bits", [8, 4])
def test_resnet50_all_layers_batch2(bits):
    """All 53 ResNet-50 conv layers (C3 shapes) at batch 2, every output byte."""
    for i, cs in enumerate(resnet50_convs(2)):
        role = cs.name.split("_")[-1]
        signed = role in ("branch2c", "branch1")
        li = make_layer_inputs(cs, bits, seed=1000 + i, relu=not signed, signed_out=signed,
                               c_store=stored_channels(cs, bits))
        _check_layer(li)


@pytest.mark.parametrize("bits", [8, 4])
def test_resnet50_batch32_sampled(bits):
    """C3 at its full batch 32 in the bench launch configuration: all outputs of two
    sampled images per layer are checked against the oracle."""
    for i, cs in enumerate(resnet50_convs(32)):
        if i % 4 and i != 52:
            continue
        role = cs.name.split("_")[-1]
        signed = role in ("branch2c", "branch1")
        li = make_layer_inputs(cs, bits, seed=2000 + i, relu=not signed, signed_out=signed,
                               c_store=stored_channels(cs, bits))
        m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
        got = _gpu_conv(li, m, n)
        for img in (0, 31):
            ref = oracle.conv2d_layer(li, mult=m, shift=n, n_slice=slice(img, img + 1))
            np.testing.assert_array_equal(got[img:img + 1], ref, err_msg=f"{cs.name} img {img}")


def test_vgg16_batch2_8bit():
    for i, cs in enumerate(vgg16_convs(2)):
        _check_layer(make_layer_inputs(cs, 8, seed=3000 + i))


# ----------------------------------------------------------------------------- C = 16 and the stem
@pytest.mark.parametrize("cs", [ConvShape("p1", 2, 9, 11, 16, 48, 3, 3, 1, 1),
                                ConvShape("p2", 1, 12, 12, 16, 64, 4, 4, 1, 0),
                                ConvShape("p3", 3, 10, 7, 16, 16, 5, 5, 2, 2),
                                ConvShape("p4", 1, 8, 8, 16, 32, 1, 1, 1, 0)], ids=lambda c: c.name)
def test_conv_c16_tap_pairs(cs):
    """8-bit C = 16: two filter taps per 32-byte K step (odd tap counts included)."""
    _check_layer(make_layer_inputs(cs, 8, seed=41))
    _check_layer(make_layer_inputs(cs, 8, seed=42, relu=False, signed_out=True))


@pytest.mark.parametrize("bits", [8, 4])
@pytest.mark.parametrize("n,x_zero", [(2, 0), (1, 3)])
def test_stem_space_to_depth(bits, n, x_zero):
    """7x7/s2/p3 C=3 stem through qconv_quantize_pack_s2d + prepare_weights_s2d + forward on
    the transformed 4x4/s1 C=16 conv, against the oracle's direct 7x7 conv."""
    from workloads import resnet50_convs
    cs = resnet50_convs(n)[0]
    rng = np.random.default_rng(100 + bits)
    xf = float_image(rng, (n, cs.h, cs.w, cs.c))
    xt = U4 if bits == 4 else U8
    s_x = 3.0 / 15 if bits == 4 else 3.0 / 255
    li = make_layer_inputs(cs, bits, seed=7 + bits, c_store=4)
    li.x_zero = x_zero
    xq = oracle.quantize(xf, s_x, x_zero, xt, c_pad=4)
    li.x_bytes = xq
    m, n_ = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n_)
    d = qc.make_desc(n, cs.h, cs.w, 3, cs.k, 7, 7, stride=2, pad=3, x_t=xt, w_t=li.w_t,
                     y_t=li.y_t, x_zero=x_zero, clamp_lo=li.clamp_lo, clamp_hi=li.clamp_hi)
    w3 = pack_codes(li.w_codes[..., :3], li.w_t) if bits == 8 else None
    if bits == 4:   # 4-bit rows of 3 channels are not byte aligned: pass 8-bit codes of s4 values
        d.w_t = S8
        w3 = pack_codes(li.w_codes[..., :3], S8)
    d2 = qc.qconv_s2d_desc(d)
    assert (d2.h, d2.w, d2.c, d2.r, d2.s) == (115, 115, 16, 4, 4)
    x2 = qc.qconv_quantize_pack_s2d(d, torch.from_numpy(xf).to(DEV), s_x)
    w2 = qc.qconv_prepare_weights_s2d(d, torch.from_numpy(np.ascontiguousarray(w3)).to(DEV))
    y = qc.qconv2d_forward(d2, x2, w2, torch.from_numpy(li.bias).to(DEV),
                           torch.from_numpy(m).to(DEV), torch.from_numpy(n_).to(DEV))
    torch.cuda.synchronize()
    np.testing.assert_array_equal(y.cpu().numpy(), ref)
