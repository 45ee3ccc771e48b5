"""Pins of the CPU oracle against things other than itself (no GPU).

Every test here checks oracle/ against what the paper and the mathematics fix:
an independent formulation (explicit im2col + matmul; 1x1 conv == GEMM),
a library routine (torch conv2d in float64, torch.quantize_per_tensor), closed
forms (identity/delta kernels, saturation, requant ties), exact rationals
(fractions.Fraction for the requant multiplier), and invariants (bias
additivity, zero-point shift, channel permutation, batch concatenation).
The map from pin to oracle function is in DESIGN.md section 3.
"""
import itertools
import math
from fractions import Fraction

import numpy as np
import pytest
import torch

import oracle
from workloads import (S4, S8, S32, U4, U8, DTYPE_RANGE, ConvShape, make_layer_inputs,
                       pack_codes, unpack_codes)


def _conv_s32(x_codes, w_codes, *, xt, wt, stride=1, pad=0, dil=1, x_zero=0, bias=None,
              w_zero=None):
    n, h, w, c = x_codes.shape
    k, r, s, _ = w_codes.shape
    y = oracle.conv2d(pack_codes(x_codes, xt), pack_codes(w_codes, wt), n=n, h=h, wd=w, c=c, k=k,
                      r=r, s=s, xt=xt, wt=wt, yt=S32, stride=(stride, stride), pad=(pad, pad),
                      dil=(dil, dil), x_zero=x_zero, bias=bias, w_zero=w_zero)
    return y.astype(np.int64)


def _im2col_matmul(x_codes, w_codes, stride, pad, dil, x_zero):
    """P:L80 explicit GEMM formulation: global im2col then one matmul (numpy int64)."""
    n, h, w, c = x_codes.shape
    k, r, s, _ = w_codes.shape
    xc = np.zeros((n, h + 2 * pad, w + 2 * pad, c), dtype=np.int64)   # padding = real zero
    xc[:, pad:pad + h, pad:pad + w, :] = x_codes - x_zero
    p = (h + 2 * pad - dil * (r - 1) - 1) // stride + 1
    q = (w + 2 * pad - dil * (s - 1) - 1) // stride + 1
    cols = np.empty((n, p, q, r, s, c), dtype=np.int64)
    for rr in range(r):
        for ss in range(s):
            cols[:, :, :, rr, ss, :] = xc[:, rr * dil: rr * dil + stride * (p - 1) + 1: stride,
                                          ss * dil: ss * dil + stride * (q - 1) + 1: stride, :]
    a = cols.reshape(n * p * q, r * s * c)
    b = w_codes.reshape(k, r * s * c)
    return (a @ b.T).reshape(n, p, q, k)


# ---------------------------------------------------------------------------- P2
@pytest.mark.parametrize("case", [
    dict(n=2, h=7, w=9, c=5, k=3, r=3, s=3, stride=1, pad=1, dil=1),
    dict(n=1, h=8, w=8, c=4, k=6, r=3, s=2, stride=2, pad=1, dil=1),
    dict(n=3, h=6, w=5, c=3, k=2, r=2, s=3, stride=1, pad=2, dil=2),
    dict(n=1, h=11, w=11, c=2, k=4, r=7, s=7, stride=2, pad=3, dil=1),
    dict(n=2, h=5, w=5, c=8, k=3, r=1, s=1, stride=2, pad=0, dil=1),
])
@pytest.mark.parametrize("bits,xt,wt", [(8, U8, S8), (8, S8, S8), (4, U4, S4), (4, S4, S4)])
def test_p2_im2col_matmul(case, bits, xt, wt):
    rng = np.random.default_rng(1)
    lo_x, hi_x = DTYPE_RANGE[xt]
    lo_w, hi_w = DTYPE_RANGE[wt]
    c = case["c"] + (case["c"] % 2 if bits == 4 else 0)
    x = rng.integers(lo_x, hi_x + 1, size=(case["n"], case["h"], case["w"], c))
    w = rng.integers(lo_w, hi_w + 1, size=(case["k"], case["r"], case["s"], c))
    zx = int(rng.integers(lo_x, hi_x + 1))
    got = _conv_s32(x, w, xt=xt, wt=wt, stride=case["stride"], pad=case["pad"], dil=case["dil"],
                    x_zero=zx)
    ref = _im2col_matmul(x, w, case["stride"], case["pad"], case["dil"], zx)
    np.testing.assert_array_equal(got, ref)


# ---------------------------------------------------------------------------- P10 lib
@pytest.mark.parametrize("stride,pad,dil", [(1, 1, 1), (2, 3, 1), (1, 2, 2), (2, 0, 1)])
def test_p10_torch_conv2d_float64(stride, pad, dil):
    rng = np.random.default_rng(2)
    x = rng.integers(0, 256, size=(2, 9, 10, 16))
    w = rng.integers(-128, 128, size=(8, 3, 3, 16))
    bias = rng.integers(-5000, 5000, size=8).astype(np.int32)
    got = _conv_s32(x, w, xt=U8, wt=S8, stride=stride, pad=pad, dil=dil, x_zero=7, bias=bias)
    xt_ = torch.from_numpy((x - 7).astype(np.float64)).permute(0, 3, 1, 2)
    wt_ = torch.from_numpy(w.astype(np.float64)).permute(0, 3, 1, 2)
    ref = torch.nn.functional.conv2d(xt_, wt_, bias=torch.from_numpy(bias.astype(np.float64)),
                                     stride=stride, padding=pad, dilation=dil)
    np.testing.assert_array_equal(got, ref.permute(0, 2, 3, 1).numpy().astype(np.int64))


# ---------------------------------------------------------------------------- P3
@pytest.mark.parametrize("xt,wt", [(U8, S8), (U4, S4), (S4, S4)])
def test_p3_1x1_is_gemm(xt, wt):
    rng = np.random.default_rng(3)
    x = rng.integers(*DTYPE_RANGE[xt], size=(2, 5, 6, 24), endpoint=True)
    w = rng.integers(*DTYPE_RANGE[wt], size=(10, 1, 1, 24), endpoint=True)
    got = _conv_s32(x, w, xt=xt, wt=wt)
    ref = x.reshape(-1, 24) @ w.reshape(10, 24).T
    np.testing.assert_array_equal(got.reshape(-1, 10), ref)


# ---------------------------------------------------------------------------- P4
@pytest.mark.parametrize("xt,yt,zx", [(U8, S8, 0), (U8, S8, 100), (U4, S4, 5), (S8, S8, 0)])
def test_p4_identity_kernel(xt, yt, zx):
    """R=S=1, K=C, W=I, bias 0, m=2^30, shift=30 (M=1), z_y=0, full clamp => Y = clamp(X - zx)."""
    rng = np.random.default_rng(4)
    c = 8
    x = rng.integers(*DTYPE_RANGE[xt], size=(1, 4, 5, c), endpoint=True)
    w = np.eye(c, dtype=np.int64).reshape(c, 1, 1, c)
    wt = S4 if xt in (U4, S4) else S8
    y = oracle.conv2d(pack_codes(x, xt), pack_codes(w, wt), n=1, h=4, wd=5, c=c, k=c, r=1, s=1,
                      xt=xt, wt=wt, yt=yt, x_zero=zx, mult=np.full(c, 1 << 30, np.int32),
                      shift=np.full(c, 30, np.int32))
    lo, hi = DTYPE_RANGE[yt]
    np.testing.assert_array_equal(unpack_codes(y, yt, c), np.clip(x - zx, lo, hi))


# ---------------------------------------------------------------------------- P5
def test_p5_delta_kernels():
    rng = np.random.default_rng(5)
    x = rng.integers(0, 256, size=(1, 7, 8, 4))
    for (rr, ss) in itertools.product(range(3), range(3)):
        w = np.zeros((4, 3, 3, 4), dtype=np.int64)
        for ch in range(4):
            w[ch, rr, ss, ch] = 1
        got = _conv_s32(x, w, xt=U8, wt=S8, pad=1)
        # shifted copy with zero borders
        ref = np.zeros_like(x)
        for p, q in itertools.product(range(7), range(8)):
            hh, ww = p - 1 + rr, q - 1 + ss
            if 0 <= hh < 7 and 0 <= ww < 8:
                ref[0, p, q] = x[0, hh, ww]
        np.testing.assert_array_equal(got, ref)
    # stride 2 subsamples, dilation 2 moves the tap
    w = np.zeros((4, 3, 3, 4), dtype=np.int64)
    for ch in range(4):
        w[ch, 2, 2, ch] = 1
    got = _conv_s32(x, w, xt=U8, wt=S8, pad=0, stride=2)
    np.testing.assert_array_equal(got, x[:, 2::2, 2::2][:, :got.shape[1], :got.shape[2]])
    got = _conv_s32(x, w, xt=U8, wt=S8, pad=0, dil=2)
    np.testing.assert_array_equal(got, x[:, 4:, 4:][:, :got.shape[1], :got.shape[2]])


# ---------------------------------------------------------------------------- P6
@pytest.mark.parametrize("xt,wt", [(U8, S8), (S8, S8), (U4, S4), (S4, S4)])
def test_p6_saturation_closed_form(xt, wt):
    lo_x, hi_x = DTYPE_RANGE[xt]
    lo_w, hi_w = DTYPE_RANGE[wt]
    r = s = 3
    c = 16
    for xv, wv in [(hi_x, hi_w), (hi_x, lo_w), (lo_x, lo_w), (lo_x, hi_w)]:
        x = np.full((1, 4, 4, c), xv)
        w = np.full((2, r, s, c), wv)
        got = _conv_s32(x, w, xt=xt, wt=wt, pad=1, bias=np.array([3, -3], np.int32))
        # interior output (1,1): all 9 taps valid; corner (0,0): 4 taps valid
        assert got[0, 1, 1, 0] == 9 * c * xv * wv + 3
        assert got[0, 0, 0, 1] == 4 * c * xv * wv - 3
        # re-quantized: clamps to the output range (M = 1)
        for yt in (U8, S8, U4, S4):
            y = oracle.conv2d(pack_codes(x, xt), pack_codes(w, wt), n=1, h=4, wd=4, c=c, k=2,
                              r=r, s=s, xt=xt, wt=wt, yt=yt, pad=(1, 1),
                              bias=np.array([3, -3], np.int32),
                              mult=np.full(2, 1 << 30, np.int32), shift=np.full(2, 30, np.int32))
            ylo, yhi = DTYPE_RANGE[yt]
            exp = np.clip(got, ylo, yhi)
            np.testing.assert_array_equal(unpack_codes(y, yt, 2), exp)
    # ReLU by truncation range: lo = max(qmin, z_y)
    x = np.full((1, 3, 3, c), hi_x)
    w = np.full((2, 1, 1, c), lo_w)
    y = oracle.conv2d(pack_codes(x, xt), pack_codes(w, wt), n=1, h=3, wd=3, c=c, k=2, r=1, s=1,
                      xt=xt, wt=wt, yt=S8, y_zero=3, clamp_lo=3, clamp_hi=127,
                      mult=np.full(2, 1 << 30, np.int32), shift=np.full(2, 30, np.int32))
    assert (unpack_codes(y, S8, 2) == 3).all()


def test_p12_overflow_is_flagged():
    """Accumulators outside int32 are outside the paper's 32-bit contract:
    the oracle refuses them instead of silently wrapping."""
    x = np.full((1, 1, 1, 64), -128)
    w = np.full((1, 3, 3, 64), -128)
    # 64*9*16384 = 9.4M fits; force overflow with a big bias
    with pytest.raises(OverflowError):
        oracle.conv2d(pack_codes(x, S8), pack_codes(w, S8), n=1, h=1, wd=1, c=64, k=1, r=3, s=3,
                      xt=S8, wt=S8, yt=S32, pad=(1, 1), bias=np.array([2 ** 31 - 100], np.int32))


# ---------------------------------------------------------------------------- P7 / Z3
def _round_half_up_exact(acc, m, n):
    return math.floor(Fraction(acc * m, 2 ** n) + Fraction(1, 2))


@pytest.mark.parametrize("m,n", [(1 << 30, 31), (1518500250, 40), (1 << 30, 1), (2147483647, 62),
                                 (1234567891, 35)])
def test_p7_requant_rounding_ties_and_values(m, n):
    """t = round-half-up(acc*m/2^n) (Z3), checked against exact rationals, including ties."""
    rng = np.random.default_rng(7)
    accs = list(rng.integers(-(2 ** 31), 2 ** 31, size=200)) + [0, 1, -1, 2 ** 31 - 1, -(2 ** 31)]
    # exact ties acc*m = (2j+1) * 2^(n-1)
    if n <= 31:
        g = math.gcd(m, 2 ** (n - 1))
        step = 2 ** (n - 1) // g
        for j in (-3, -1, 0, 1, 5):
            acc = (2 * j + 1) * step
            if -(2 ** 31) <= acc < 2 ** 31 and (acc * m) % (2 ** n) == 2 ** (n - 1):
                accs.append(acc)
    accs = np.array(accs, dtype=np.int64)
    # acc_pure = bias (1x1 conv with zero input): y = clamp(t) with huge clamp via s32-free path
    k = len(accs)
    x = np.zeros((1, 1, 1, 32), dtype=np.int64)
    w = np.zeros((k, 1, 1, 32), dtype=np.int64)
    # S8 output saturates; compare only where the exact value is in range, and the clamp elsewhere
    y = oracle.conv2d(pack_codes(x, U8), pack_codes(w, S8), n=1, h=1, wd=1, c=32, k=k, r=1, s=1,
                      xt=U8, wt=S8, yt=S8, bias=accs.astype(np.int32),
                      mult=np.full(k, m, np.int32), shift=np.full(k, n, np.int32))
    got = unpack_codes(y, S8, k)[0, 0, 0]
    exp = np.array([min(127, max(-128, _round_half_up_exact(int(a), m, n))) for a in accs])
    np.testing.assert_array_equal(got, exp)


def test_p7_tie_direction():
    """acc*m = -2^(n-1) rounds to 0 (toward +inf); +2^(n-1) rounds to 1."""
    x = np.zeros((1, 1, 1, 32), dtype=np.int64)
    w = np.zeros((2, 1, 1, 32), dtype=np.int64)
    y = oracle.conv2d(pack_codes(x, U8), pack_codes(w, S8), n=1, h=1, wd=1, c=32, k=2, r=1, s=1,
                      xt=U8, wt=S8, yt=S8, bias=np.array([-1, 1], np.int32),
                      mult=np.full(2, 1 << 30, np.int32), shift=np.full(2, 31, np.int32))
    assert list(unpack_codes(y, S8, 2)[0, 0, 0]) == [0, 1]
    y = oracle.conv2d(pack_codes(x, U8), pack_codes(w, S8), n=1, h=1, wd=1, c=32, k=2, r=1, s=1,
                      xt=U8, wt=S8, yt=S8, bias=np.array([-3, 3], np.int32),
                      mult=np.full(2, 1 << 30, np.int32), shift=np.full(2, 31, np.int32))
    assert list(unpack_codes(y, S8, 2)[0, 0, 0]) == [-1, 2]


# ---------------------------------------------------------------------------- P8 (R1)
def test_p8_requant_params_exact():
    rng = np.random.default_rng(8)
    s_in = np.float32(0.0173)
    s_w = np.concatenate([rng.uniform(1e-4, 0.1, 300).astype(np.float32),
                          np.float32([0.0, 1.0, 0.5, 2.0 ** -20])])
    s_out = np.float32(0.0421)
    m, n = oracle.requant_params(s_in, s_w, s_out)
    for i, sw in enumerate(s_w):
        if sw == 0:
            assert m[i] == 0 and n[i] == 31
            continue
        M = Fraction(float(s_in)) * Fraction(float(sw)) / Fraction(float(s_out))
        approx = Fraction(int(m[i]), 2 ** int(n[i]))
        assert 2 ** 30 <= m[i] < 2 ** 31
        e = int(n[i])  # M ~ m*2^-n, m in [2^30, 2^31): half-ulp of the 31-bit mantissa = 2^-(n+1)
        # RNE division (rel. 2^-53) + half-up mantissa rounding (<= 2^-(n+1)), exactly bounded:
        assert abs(approx - M) <= Fraction(1, 2 ** (e + 1)) + M * Fraction(1, 2 ** 52)


def test_p8_requant_params_edges():
    # M = 1 -> (2^30, 30); M = 0.5 -> (2^30, 31); M = 3 -> (3*2^29, 29)
    m, n = oracle.requant_params(1.0, np.float32([1.0, 0.5, 3.0]), 1.0)
    assert list(m) == [2 ** 30, 2 ** 30, 3 * 2 ** 29] and list(n) == [30, 31, 29]
    # M = 1/(1+2^-23) = 1 - 2^-23 + 2^-46 - ... -> f*2^31 = 2^31 - 2^8 + 2^-15.. -> m = 2^31-256
    m2, n2 = oracle.requant_params(np.float32(1.0), np.float32([1.0]), np.float32(1.0 + 2 ** -23))
    assert m2[0] == 2 ** 31 - 256 and n2[0] == 31
    # tiny M (shift > 62) and non-positive scales are rejected
    with pytest.raises(ValueError):
        oracle.requant_params(1e-10, np.float32([1e-10]), 1.0)
    with pytest.raises(ValueError):
        oracle.requant_params(-1.0, np.float32([1.0]), 1.0)


def test_p8_renormalisation_branch():
    """a*b/c = 1 - 2^-46/c: f*2^31 rounds up to 2^31 and must renormalise to (2^30, 30).
    a = 1+3u, b = 1+5592405u, c = 1+5592410u (u = 2^-23): 3*5592405 = 2*2^23 - 1."""
    u = 2.0 ** -23
    a, b, c = np.float32(1 + 3 * u), np.float32(1 + 5592405 * u), np.float32(1 + 5592410 * u)
    M = Fraction(float(a)) * Fraction(float(b)) / Fraction(float(c))
    assert 1 - Fraction(1, 2 ** 40) < M < 1
    m, n = oracle.requant_params(a, np.float32([b]), c)
    assert m[0] == 2 ** 30 and n[0] == 30


# ---------------------------------------------------------------------------- P9
@pytest.mark.parametrize("scale,zp", [(0.0173, 0), (0.25, 3), (1.0, 0), (3.0 / 15, 0), (0.0071, 7)])
def test_p9_quantize_vs_torch(scale, zp):
    rng = np.random.default_rng(9)
    x = np.concatenate([rng.normal(0, 2, 20000), rng.normal(0, 50 * scale, 20000),
                        # exact ties of x * fl32(1/s)
                        (np.arange(-300, 300) + 0.5) * scale,
                        [np.inf, -np.inf, 0.0, -0.0, 1e30, -1e30, 7.0, -7.0]]).astype(np.float32)
    x = x.reshape(-1, 4)
    xt = torch.from_numpy(x)
    q_u8 = torch.quantize_per_tensor(xt, scale, zp, torch.quint8).int_repr().numpy().astype(np.int64)
    got = unpack_codes(oracle.quantize(x, scale, zp, U8), U8, 4)
    np.testing.assert_array_equal(got, q_u8)
    q_s8 = torch.quantize_per_tensor(xt, scale, zp, torch.qint8).int_repr().numpy().astype(np.int64)
    np.testing.assert_array_equal(unpack_codes(oracle.quantize(x, scale, zp, S8), S8, 4), q_s8)
    # 4-bit = clamp of the 8-bit code (the 4-bit range is inside the 8-bit range)
    if zp <= 7:
        np.testing.assert_array_equal(unpack_codes(oracle.quantize(x, scale, zp, U4), U4, 4),
                                      np.clip(q_u8, 0, 15))
        np.testing.assert_array_equal(unpack_codes(oracle.quantize(x, scale, zp, S4), S4, 4),
                                      np.clip(q_s8, -8, 7))


def test_p9_quantize_bf16_pad_nan():
    rng = np.random.default_rng(10)
    xf = torch.from_numpy(rng.normal(0, 1, (3, 5, 6)).astype(np.float32)).to(torch.bfloat16)
    bits = xf.view(torch.int16).numpy().view(np.uint16)
    got = oracle.quantize(bits, 0.05, 4, U4, c_pad=8, bf16=True)
    ref = torch.quantize_per_tensor(xf.float(), 0.05, 4, torch.quint8).int_repr().numpy()
    codes = unpack_codes(got, U4, 8)
    np.testing.assert_array_equal(codes[..., :6], np.clip(ref.astype(np.int64), 0, 15))
    assert (codes[..., 6:] == 4).all()      # padded channels hold the zero point
    # NaN -> zero point (reading Z4)
    xn = np.full((1, 2), np.nan, np.float32)
    assert (unpack_codes(oracle.quantize(xn, 0.1, 9, U8), U8, 2) == 9).all()
    # nibble order (Z7): element 2j in the low nibble of byte j
    one = np.array([[1.0, 2.0]], np.float32)
    assert oracle.quantize(one, 1.0, 0, U4)[0, 0] == 0x21


# ---------------------------------------------------------------------------- P10 invariants
def test_p10_invariants():
    rng = np.random.default_rng(11)
    x = rng.integers(0, 200, size=(3, 6, 7, 16))
    w = rng.integers(-120, 121, size=(5, 3, 3, 16))
    base = _conv_s32(x, w, xt=U8, wt=S8, pad=1)
    # bias additivity
    b = rng.integers(-1000, 1000, size=5).astype(np.int32)
    np.testing.assert_array_equal(_conv_s32(x, w, xt=U8, wt=S8, pad=1, bias=b), base + b)
    # shifting X and z_x together leaves the result unchanged (borders included)
    np.testing.assert_array_equal(_conv_s32(x + 40, w, xt=U8, wt=S8, pad=1, x_zero=40), base)
    # K-permutation equivariance
    perm = rng.permutation(5)
    np.testing.assert_array_equal(_conv_s32(x, w[perm], xt=U8, wt=S8, pad=1), base[..., perm])
    # batch concatenation (the multi-GPU sharding argument)
    parts = [_conv_s32(x[i:i + 1], w, xt=U8, wt=S8, pad=1) for i in range(3)]
    np.testing.assert_array_equal(np.concatenate(parts, axis=0), base)
    # per-channel weight zero point == subtracting it from the weights
    zw = rng.integers(-3, 4, size=5).astype(np.int32)
    np.testing.assert_array_equal(_conv_s32(x, w, xt=U8, wt=S8, pad=1, w_zero=zw),
                                  _conv_s32(x, w - zw.reshape(5, 1, 1, 1), xt=U8, wt=S8, pad=1))


def test_p10_requant_close_to_real_multiplier():
    """y ~ round(acc * s_x s_w / s_y): the integer epilogue is within 1/2 + |acc| eps."""
    li = make_layer_inputs(ConvShape("t", 2, 9, 9, 32, 16, 3, 3, 1, 1), 8, seed=3, relu=False,
                           signed_out=True)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    acc = oracle.conv2d_layer(li, y_t=S32).astype(np.int64)
    y = unpack_codes(oracle.conv2d_layer(li, mult=m, shift=n), li.y_t, 16)
    M = (np.float64(li.s_x) * li.s_w.astype(np.float64)) / np.float64(li.s_y)
    real = np.clip(acc * M, -128, 127)
    assert np.max(np.abs(y - real)) <= 0.5 + 1e-6 * np.max(np.abs(acc) + 1)


# ---------------------------------------------------------------------------- P1 brute force
def test_p1_exhaustive_tiny_4bit():
    """Every signed 4-bit (x, w) pair through a 1x1 conv (pixels carry x, output channels
    carry w): y = clamp(round-half-up(x*w*m/2^n)) against exact rationals."""
    xs = np.arange(-8, 8)
    ws = np.arange(-8, 8)
    x = np.zeros((1, 1, 16, 2), dtype=np.int64)
    x[0, 0, :, 0] = xs
    w = np.zeros((16, 1, 1, 2), dtype=np.int64)
    w[:, 0, 0, 0] = ws
    for m, n in [(1 << 30, 30), (1288490189, 33), (1 << 30, 32), (1 << 30, 28)]:
        y = oracle.conv2d(pack_codes(x, S4), pack_codes(w, S4), n=1, h=1, wd=16, c=2, k=16, r=1,
                          s=1, xt=S4, wt=S4, yt=S8, mult=np.full(16, m, np.int32),
                          shift=np.full(16, n, np.int32))
        got = unpack_codes(y, S8, 16)[0, 0]
        exp = np.array([[_round_half_up_exact(int(a) * int(b), m, n) for b in ws] for a in xs])
        np.testing.assert_array_equal(got, np.clip(exp, -128, 127))


# ---------------------------------------------------------------------------- P13 (Z15)
def _round_half_away_exact(fr: Fraction) -> int:
    """Nearest integer, ties away from zero (what gemmlowp documents RoundingDivideByPOT to do)."""
    a = abs(fr)
    r = math.floor(a + Fraction(1, 2))
    return r if fr >= 0 else -r


def test_p13_gemmlowp_primitives_documented_values():
    """Values fixed by gemmlowp's documentation of the two primitives (Q31 products, ties of
    the divide away from zero) and the one saturating case."""
    assert oracle.srdhm(1 << 30, 1 << 30) == 1 << 29            # 0.5 * 0.5 = 0.25 in Q31
    assert oracle.srdhm(-(1 << 31), -(1 << 31)) == 2 ** 31 - 1  # saturation
    assert oracle.srdhm(2 ** 31 - 1, 2 ** 31 - 1) == 2 ** 31 - 2
    assert oracle.srdhm(-(1 << 31), 1 << 30) == -(1 << 30)
    assert [oracle.rdbpot(v, 1) for v in (5, -5, 3, -3, 4, -4, 1, -1)] == [3, -3, 2, -2, 2, -2, 1, -1]
    assert oracle.rdbpot(-(1 << 31), 31) == -1 and oracle.rdbpot(2 ** 31 - 1, 31) == 1
    assert oracle.rdbpot(12345, 0) == 12345


def test_p13_gemmlowp_primitives_vs_exact_rationals():
    """SRDHM(a,b) = round-half-up(a*b / 2^31) and RDBPOT(x,e) = round-half-away(x / 2^e),
    checked against exact rationals on random and tie-constructing operands."""
    rng = np.random.default_rng(13)
    lim = 2 ** 31
    a = list(rng.integers(-lim, lim, 3000)) + [0, 1, -1, lim - 1, -lim, 1 << 30, -(1 << 30)]
    b = list(rng.integers(-lim, lim, 3000)) + [lim - 1, lim - 1, lim - 1, 1, 1, 3, 3]
    for x, y in zip(a, b):
        x, y = int(x), int(y)
        if x == -lim and y == -lim:
            continue
        exp = math.floor(Fraction(x * y, 2 ** 31) + Fraction(1, 2))
        assert oracle.srdhm(x, y) == exp, (x, y)
    for e in (0, 1, 2, 5, 13, 30, 31):
        xs = list(rng.integers(-lim, lim, 300)) + [((2 * j + 1) << e) // 2 for j in range(-4, 4)
                                                   if e > 0 and -lim <= ((2 * j + 1) << e) // 2 < lim]
        for x in xs:
            x = int(x)
            assert oracle.rdbpot(x, e) == _round_half_away_exact(Fraction(x, 2 ** e)), (x, e)


@pytest.mark.parametrize("m,sh", [(1 << 30, 31), (1518500250, 40), (1 << 30, 29), (2147483647, 62),
                                  (1234567891, 35), (1 << 30, 1), (1 << 30, 33)])
def test_p13_tflite_requant_through_conv(m, sh):
    """rounding = 1 through the conv (acc = bias of a zero-input 1x1 conv): y = clamp(RDBPOT(
    SRDHM(sat32(acc * 2^ls), m), rs)) with ls/rs from the TFLite exponent 31 - shift, each
    step as an exact rational; and the single-rounding result differs on constructed ties."""
    rng = np.random.default_rng(sh)
    accs = np.array(list(rng.integers(-(2 ** 31), 2 ** 31, size=300)) + [0, 1, -1, 2 ** 31 - 1,
                                                                        -(2 ** 31)], np.int64)
    k = len(accs)
    x = np.zeros((1, 1, 1, 32), dtype=np.int64)
    w = np.zeros((k, 1, 1, 32), dtype=np.int64)
    y = oracle.conv2d(pack_codes(x, U8), pack_codes(w, S8), n=1, h=1, wd=1, c=32, k=k, r=1, s=1,
                      xt=U8, wt=S8, yt=S8, bias=accs.astype(np.int32), rounding=1,
                      mult=np.full(k, m, np.int32), shift=np.full(k, sh, np.int32))
    got = unpack_codes(y, S8, k)[0, 0, 0]
    ls, rs = max(0, 31 - sh), max(0, sh - 31)
    exp = []
    for acc in accs:
        a = min(2 ** 31 - 1, max(-(2 ** 31), int(acc) * 2 ** ls))
        hm = math.floor(Fraction(a * m, 2 ** 31) + Fraction(1, 2))
        exp.append(min(127, max(-128, _round_half_away_exact(Fraction(hm, 2 ** rs)))))
    np.testing.assert_array_equal(got, np.array(exp))


def test_p13_double_rounding_differs_from_single():
    """acc*m/2^n = -2.5 exactly: single rounding (ties toward +inf) gives -2, the TFLite
    double rounding (SRDHM exact here, RDBPOT ties away from zero) gives -3."""
    m, sh = 1 << 30, 33                       # M = 2^-3: acc = -20 -> -2.5
    x = np.zeros((1, 1, 1, 32), dtype=np.int64)
    w = np.zeros((2, 1, 1, 32), dtype=np.int64)
    kw = dict(n=1, h=1, wd=1, c=32, k=2, r=1, s=1, xt=U8, wt=S8, yt=S8,
              bias=np.array([-20, 20], np.int32), mult=np.full(2, m, np.int32),
              shift=np.full(2, sh, np.int32))
    single = unpack_codes(oracle.conv2d(pack_codes(x, U8), pack_codes(w, S8), **kw), S8, 2)
    tfl = unpack_codes(oracle.conv2d(pack_codes(x, U8), pack_codes(w, S8), rounding=1, **kw), S8, 2)
    assert list(single[0, 0, 0]) == [-2, 3] and list(tfl[0, 0, 0]) == [-3, 3]


# ---------------------------------------------------------------------------- P14 (Z16)
@pytest.mark.parametrize("relu", [False, True])
def test_p14_dequant_output_vs_numpy_and_torch(relu):
    """Fusion of convolution and dequantization: y = fl32(fl32(acc) * scale[k]).
    Checked against numpy's IEEE float32 product of the int32 result (a library routine, not
    the oracle's own arithmetic) and, for bf16, torch's round-to-nearest-even conversion."""
    from oracle import BF16, F32
    li = make_layer_inputs(ConvShape("dq", 2, 9, 8, 32, 24, 3, 3, 1, 1), 8, seed=14, relu=False,
                           signed_out=True)
    li.bias[:4] = [2 ** 24 + 1, -(2 ** 24 + 3), 2 ** 30, -(2 ** 30)]   # int->fp32 rounding cases
    acc = oracle.conv2d_layer(li, y_t=S32)
    scale = (np.float32(li.s_x) * li.s_w).astype(np.float32)
    ref = acc.astype(np.float32) * scale
    if relu:
        ref = np.where(ref > 0, ref, np.float32(0.0))
    got = oracle.conv2d_layer(li, y_t=F32, dq_scale=scale, relu=relu)
    assert got.dtype == np.float32
    np.testing.assert_array_equal(got.view(np.uint32), ref.view(np.uint32))   # bit-exact, +0 only
    gotb = oracle.conv2d_layer(li, y_t=BF16, dq_scale=scale, relu=relu)
    refb = torch.from_numpy(ref).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    np.testing.assert_array_equal(gotb, refb)
