"""GPU parity for the data paths added in round 1's optimisation pass, each forced onto the
kernel that owns it (`qconv.cu: qconv2d_forward` kernel choice):

* channel-major 1x1 kernel (`qconv_t_kernel`, K % 64 == 0): the channel-pair epilogue in its
  fast / mid / general requant modes, M = 64 and M = 128 tiles, 4- and 8-bit outputs, signed
  and unsigned, ReLU6-style clamps;
* nibble-plane 4-bit widening with SIGNED activations (the +8 offset and the per-channel
  weight-sum correction) in all three kernels;
* 4-bit layers whose effective bias leaves the fast/mid range (|b_eff| >= 2^26: the general
  mode shifts the x16 accumulator back first).

Every comparison is byte equality with the CPU oracle (P:L273 exactness).
"""
import numpy as np
import pytest

import oracle
from workloads import (S4, S8, U4, U8, ConvShape, DTYPE_RANGE, make_layer_inputs, pack_codes)

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA GPU", allow_module_level=True)

import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc  # noqa: E402

DEV = "cuda:0"


def _run(li, m, n, y_t=None, lo=None, hi=None):
    cs = li.shape
    yt = li.y_t if y_t is None else y_t
    clo = li.clamp_lo if lo is None else lo
    chi = li.clamp_hi if hi is None else hi
    d = qc.make_desc(cs.n, cs.h, cs.w, li.x_codes.shape[-1], cs.k, cs.r, cs.s, stride=cs.stride,
                     pad=cs.pad, dil=cs.dil, x_t=li.x_t, w_t=li.w_t, y_t=yt, x_zero=li.x_zero,
                     y_zero=li.y_zero, clamp_lo=clo, clamp_hi=chi)
    x = torch.from_numpy(li.x_bytes).to(DEV)
    w = torch.from_numpy(li.w_bytes).to(DEV)
    b = torch.from_numpy(li.bias).to(DEV)
    y = qc.qconv2d_forward(d, x, w, b, torch.from_numpy(m).to(DEV), torch.from_numpy(n).to(DEV))
    torch.cuda.synchronize()
    return y.cpu().numpy()


def _check(li, m, n, lo=None, hi=None):
    if lo is not None:
        li.clamp_lo, li.clamp_hi = lo, hi
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    got = _run(li, m, n)
    if not np.array_equal(got, ref):
        bad = np.argwhere(got != ref)
        raise AssertionError(f"{bad.shape[0]} mismatching bytes of {ref.size}; first {bad[:5]}")


def _signed_inputs(li, bits, rng):
    """Replace the activations by signed codes over the full range (extremes included)."""
    xt = S4 if bits == 4 else S8
    lo, hi = DTYPE_RANGE[xt]
    li.x_t = xt
    li.x_codes = rng.integers(lo, hi + 1, size=li.x_codes.shape)
    li.x_codes.reshape(-1, li.x_codes.shape[-1])[:5] = lo
    li.x_codes.reshape(-1, li.x_codes.shape[-1])[5:9] = hi
    li.x_bytes = pack_codes(li.x_codes, xt)
    return li


# 1x1 shapes that take the channel-major kernel: K = 64 (M64 tiles), K = 128, K = 192 (both)
T_SHAPES = [ConvShape("t64", 2, 12, 13, 64, 64, 1, 1),
            ConvShape("t128", 1, 20, 20, 128, 128, 1, 1, 2, 0),
            ConvShape("t192", 3, 9, 10, 256, 192, 1, 1)]


@pytest.mark.parametrize("cs", T_SHAPES, ids=lambda c: c.name)
@pytest.mark.parametrize("bits", [4, 8])
@pytest.mark.parametrize("lo_n,hi_n", [(33, 52), (20, 33), (14, 60)])
def test_channel_major_requant_modes(cs, bits, lo_n, hi_n):
    """fast (33..52), mid (20..33) and general (outside both) epilogue modes of the pair
    epilogue, with signed outputs that saturate both ways."""
    li = make_layer_inputs(cs, bits, seed=lo_n * 3 + bits + cs.k, relu=False, signed_out=True)
    rng = np.random.default_rng(lo_n + hi_n + cs.k)
    m = rng.integers(1 << 30, 1 << 31, size=cs.k).astype(np.int32)
    n = rng.integers(lo_n, hi_n + 1, size=cs.k).astype(np.int32)
    _check(li, m, n)


@pytest.mark.parametrize("cs", T_SHAPES, ids=lambda c: c.name)
@pytest.mark.parametrize("bits", [4, 8])
def test_channel_major_signed_inputs_and_clamp(cs, bits):
    rng = np.random.default_rng(cs.k + bits)
    li = _signed_inputs(make_layer_inputs(cs, bits, seed=31 + bits, relu=True), bits, rng)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    _check(li, m, n)
    qhi = DTYPE_RANGE[li.y_t][1]
    _check(li, m, n, lo=1, hi=min(qhi, 6))              # ReLU6-style truncation range


@pytest.mark.parametrize("cs", [ConvShape("halo", 2, 12, 14, 64, 64, 3, 3, 1, 1),
                                ConvShape("im2col", 2, 9, 9, 96, 48, 3, 3, 2, 1),
                                ConvShape("one", 1, 16, 16, 256, 128, 1, 1)],
                         ids=lambda c: c.name)
def test_signed_int4_activations_every_kernel(cs):
    """Signed 4-bit activations are widened as x + 8 and corrected by 8 * sum_w (nibble-plane
    widening); OOB padding must still count as 0."""
    rng = np.random.default_rng(cs.c + cs.k)
    li = _signed_inputs(make_layer_inputs(cs, 4, seed=77, relu=False, signed_out=True), 4, rng)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    _check(li, m, n)


@pytest.mark.parametrize("cs", [ConvShape("halo", 1, 10, 10, 64, 64, 3, 3, 1, 1),
                                ConvShape("t", 1, 8, 8, 64, 128, 1, 1),
                                ConvShape("im2col", 1, 9, 9, 64, 32, 3, 3, 2, 1)],
                         ids=lambda c: c.name)
def test_int4_large_bias_general_mode(cs):
    """|bias| >= 2^26 leaves the x16 fast/mid range: those chunks take the general mode."""
    li = make_layer_inputs(cs, 4, seed=5, relu=False, signed_out=True)
    rng = np.random.default_rng(9)
    li.bias[: cs.k // 2] = rng.integers(1 << 26, 1 << 27, size=cs.k // 2) * rng.choice([-1, 1], size=cs.k // 2)
    m = rng.integers(1 << 30, 1 << 31, size=cs.k).astype(np.int32)
    n = rng.integers(40, 50, size=cs.k).astype(np.int32)
    _check(li, m, n)


# ----------------------------------------------------------------------------- CTA-pair kernel
@pytest.mark.parametrize("cs", [ConvShape("res4_3x3_b100", 100, 14, 14, 256, 256, 3, 3, 1, 1),
                                ConvShape("res5_3x3_b400", 400, 7, 7, 512, 512, 3, 3, 1, 1)],
                         ids=lambda c: c.name)
def test_cta_pair_8bit_3x3_full_tiles(cs):
    """8-bit 3x3 layers big enough for full N = 256 tiles take the CTA-pair kernel
    (fwd2.cuh, cta_group::2): every output of three sampled images (first, last, one in
    the middle -- each 256-pixel pair tile spans image boundaries) against the oracle."""
    li = make_layer_inputs(cs, 8, seed=cs.n, relu=True)
    m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
    got = _run(li, m, n)
    for img in (0, cs.n // 2 + 1, cs.n - 1):
        ref = oracle.conv2d_layer(li, mult=m, shift=n, n_slice=slice(img, img + 1))
        np.testing.assert_array_equal(got[img:img + 1], ref, err_msg=f"{cs.name} img {img}")


@pytest.mark.parametrize("bits", [8, 4])
def test_cta_pair_forced_every_eligible_layer(bits):
    """Force the CTA-pair kernel (through the plan API) onto every ResNet-50 layer at batch 2
    where it is eligible, 4-bit included, with the widest N tile it takes."""
    from workloads import resnet50_convs, stored_channels
    n_forced = 0
    for i, cs in enumerate(resnet50_convs(2)):
        li = make_layer_inputs(cs, bits, seed=4000 + i, relu=True, c_store=stored_channels(cs, bits))
        d = qc.make_desc(cs.n, cs.h, cs.w, li.x_codes.shape[-1], cs.k, cs.r, cs.s, stride=cs.stride,
                         pad=cs.pad, x_t=li.x_t, w_t=li.w_t, y_t=li.y_t, clamp_lo=li.clamp_lo,
                         clamp_hi=li.clamp_hi)
        pairs = [c for c in qc.qconv_plan_candidates(d) if c["kernel"] == qc.QC_KERNEL_PAIR]
        if not pairs:
            continue
        bn = max(c["bn"] for c in pairs)
        m, n = oracle.requant_params(li.s_x, li.s_w, li.s_y)
        qc.qconv_plan_set(d, qc.QC_KERNEL_PAIR, bn)
        try:
            assert qc.qconv_debug_plan(d)["kernel"] == qc.QC_KERNEL_PAIR
            got = _run(li, m, n)
        finally:
            qc.qconv_plan_set(d, None)
        ref = oracle.conv2d_layer(li, mult=m, shift=n)
        np.testing.assert_array_equal(got, ref, err_msg=f"{cs.name} pair bn={bn}")
        n_forced += 1
    assert n_forced >= 20
