"""Boundary tests that need no GPU: the C-ABI library loads, exports every symbol
include/qconv.h declares, rejects bad arguments on the host before touching the
device, and its host-only requant-parameter derivation is bit-exact with the
oracle's (reading R1)."""
import ctypes
import os
import re

import numpy as np
import pytest

import oracle
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "qconv.h")


def _declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"\b(qconv[a-z0-9_]*)\s*\(", src)
    return sorted(set(names))


def test_header_symbols_exported():
    names = _declared_functions()
    assert {"qconv_quantize_pack", "qconv_requant_params", "qconv2d_forward"} <= set(names)
    lib = ctypes.CDLL(qc.lib_path())
    for n in names:
        assert hasattr(lib, n), f"{n} declared in qconv.h but not exported"


def test_status_strings_and_version():
    lib = qc._lib()
    for s in range(7):
        assert lib.qconv_status_string(s)
    assert lib.qconv_version() >= 100


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_requant_params_match_oracle(seed):
    rng = np.random.default_rng(seed)
    s_w = np.concatenate([rng.uniform(1e-5, 0.5, 500), [0.0, 1.0, 0.5, 3.0]]).astype(np.float32)
    for s_in, s_out in [(0.05, 0.02), (0.0173, 0.0421), (1.0, 1.0), (0.2, 0.01)]:
        m1, n1 = qc.qconv_requant_params(s_in, s_w, s_out)
        m2, n2 = oracle.requant_params(s_in, s_w, s_out)
        np.testing.assert_array_equal(m1, m2)
        np.testing.assert_array_equal(n1, n2)


def test_requant_params_renormalisation_and_errors():
    u = 2.0 ** -23
    a, b, c = np.float32(1 + 3 * u), np.float32(1 + 5592405 * u), np.float32(1 + 5592410 * u)
    m, n = qc.qconv_requant_params(a, np.float32([b]), c)
    assert m[0] == 2 ** 30 and n[0] == 30
    with pytest.raises(qc.QConvError):
        qc.qconv_requant_params(-1.0, np.float32([1.0]), 1.0)
    with pytest.raises(qc.QConvError):
        qc.qconv_requant_params(1e-10, np.float32([1e-10]), 1.0)


FAKE = 1 << 20      # aligned, never dereferenced: validation fails first


def _fwd(d, x=FAKE, w=FAKE, bias=None, m=FAKE, s=FAKE, y=FAKE, ws=None, wsb=0):
    return qc._lib().qconv2d_forward(ctypes.byref(d), x, w, bias, m, s, y, ws, wsb, None)


def test_forward_host_validation():
    good = dict(n=1, h=8, w=8, c=64, k=64, r=3, s=3, pad=1)
    assert _fwd(qc.make_desc(**{**good, "c": 0})) == 1                      # INVALID_ARG
    assert _fwd(qc.make_desc(**{**good, "r": 11})) == 1                     # P < 1
    assert _fwd(qc.make_desc(**good, x_t=qc.QC_S32)) == 1                   # bad input dtype
    assert _fwd(qc.make_desc(**good, clamp_lo=10, clamp_hi=5)) == 1
    assert _fwd(qc.make_desc(**good, y_zero=300)) == 1
    assert _fwd(qc.make_desc(**good, rounding=2)) == 1
    assert _fwd(qc.make_desc(**good, y_t=qc.QC_F32_OUT)) == 1               # float: dequant call
    assert _fwd(qc.make_desc(**good), x=None) == 1
    assert _fwd(qc.make_desc(**good), m=None) == 1                          # requant ptrs needed
    assert _fwd(qc.make_desc(**{**good, "c": 3}, x_t=qc.QC_U4, w_t=qc.QC_S4)) == 1  # odd 4-bit rows
    # channel counts the kernels do not take directly are rearranged into the workspace
    d48 = qc.make_desc(**{**good, "c": 48})
    assert qc.qconv2d_workspace_size(d48) == 64 * 9 * 64 + 8 * 8 * 64      # padded w + activations
    assert qc.qconv_prepared_weight_bytes(d48) == 64 * 9 * 64
    assert _fwd(d48) == 5                                                   # WORKSPACE
    assert qc.qconv_debug_plan(d48)["prologue"] == 1 | 2
    assert _fwd(qc.make_desc(**good, x_t=qc.QC_U4, w_t=qc.QC_S8)) == 2      # A4W8
    assert _fwd(qc.make_desc(**{**good, "k": 63}, x_t=qc.QC_U4, w_t=qc.QC_S4,
                             y_t=qc.QC_U4)) == 2                            # odd K, 4-bit out
    assert _fwd(qc.make_desc(**{**good, "stride": 9})) == 2
    assert _fwd(qc.make_desc(n=1, h=8, w=8, c=64 * 1024, k=8, r=3, s=3, pad=1)) == 3  # overflow
    assert _fwd(qc.make_desc(**good), x=FAKE + 8) == 4                      # MISALIGNED
    d = qc.make_desc(**good, x_zero=3)
    assert qc.qconv2d_workspace_size(d) == 64 * 16 * 4
    assert _fwd(d) == 5                                                     # WORKSPACE
    d4 = qc.make_desc(**good, x_t=qc.QC_U4, w_t=qc.QC_S4, y_t=qc.QC_U4)
    # prepared 4-bit weights: nibble-plane int8 KRSC + int32 per-channel weight sums
    assert qc.qconv2d_workspace_size(d4) == 64 * 9 * 64 + 256              # unprepared 4-bit w
    d4.w_prepared = 1
    assert qc.qconv2d_workspace_size(d4) == 0
    assert qc.qconv_prepared_weight_bytes(d4) == 64 * 9 * 64 + 4 * 64
    # A8W4: 4-bit weights widened to int8 (no weight sums)
    da = qc.make_desc(**good, x_t=qc.QC_U8, w_t=qc.QC_S4)
    assert qc.qconv_prepared_weight_bytes(da) == 64 * 9 * 64
    assert qc.qconv2d_workspace_size(da) == 64 * 9 * 64
    # weight zero points: per-pixel activation sums in the workspace, im2col kernel
    dz = qc.make_desc(**good, w_zero=FAKE)
    assert qc.qconv2d_workspace_size(dz) == 256 + 256
    assert qc.qconv_debug_plan(dz)["kernel_name"] == "im2col"
    assert _fwd(dz) == 5


def test_plans_on_the_host():
    """Kernel choice, candidates and the plan cache need no GPU (no launch)."""
    qc.qconv_plan_clear()
    d = qc.make_desc(256, 14, 14, 256, 256, 3, 3, pad=1, x_t=qc.QC_U4, w_t=qc.QC_S4,
                     y_t=qc.QC_U4, w_prepared=1)
    assert qc.qconv_debug_plan(d)["kernel_name"] == "pair"
    cands = qc.qconv_plan_candidates(d)
    names = {(c["kernel_name"], c["bn"]) for c in cands}
    assert ("im2col", 256) in names and ("pair", 256) in names and ("im2col", 64) in names
    qc.qconv_plan_set(d, qc.QC_KERNEL_IM2COL, 128)
    p = qc.qconv_debug_plan(d)
    assert (p["kernel_name"], p["bn"]) == ("im2col", 128)
    with pytest.raises(qc.QConvError):
        qc.qconv_plan_set(d, qc.QC_KERNEL_CHANNEL, 128)                      # 3x3: ineligible
    qc.qconv_plan_set(d, None)
    assert qc.qconv_debug_plan(d)["kernel_name"] == "pair"
    # 1x1 -> channel-major; stem in s2d form (K = 64) -> channel-major halo; int32 output -> im2col
    d1 = qc.make_desc(32, 56, 56, 64, 256, 1, 1, x_t=qc.QC_U4, w_t=qc.QC_S4, y_t=qc.QC_S4,
                      w_prepared=1)
    assert qc.qconv_debug_plan(d1)["kernel_name"] == "channel"
    stem = qc.make_desc(8, 224, 224, 3, 64, 7, 7, stride=2, pad=3, w_prepared=1)
    ps = qc.qconv_debug_plan(stem)
    assert ps["kernel_name"] == "halo_t" and ps["prologue"] == 2
    assert ps["threads"] == 640 and ps["tmem_cols"] == 512 and ps["bm"] == 240   # 2 rows of 120 pixels
    qc.qconv_plan_set(stem, qc.QC_KERNEL_HALO, 0)                                 # the pixel-major one
    assert qc.qconv_debug_plan(stem)["kernel_name"] == "halo"
    qc.qconv_plan_set(stem, None)
    d32 = qc.make_desc(2, 9, 9, 64, 48, 3, 3, pad=1, y_t=qc.QC_S32)
    assert qc.qconv_debug_plan(d32)["kernel_name"] == "im2col"


def test_quantize_host_validation():
    L = qc._lib()
    assert L.qconv_quantize_pack(FAKE, 0, 10, 3, 2, 1.0, 0, qc.QC_U8, FAKE, None) == 1   # c_pad<c
    assert L.qconv_quantize_pack(FAKE, 0, 10, 3, 3, 1.0, 0, qc.QC_U4, FAKE, None) == 1   # odd pad
    assert L.qconv_quantize_pack(FAKE, 0, 10, 4, 4, -1.0, 0, qc.QC_U8, FAKE, None) == 1
    assert L.qconv_quantize_pack(FAKE, 0, 10, 4, 4, 1.0, 16, qc.QC_U4, FAKE, None) == 1  # zp
    assert L.qconv_quantize_pack(FAKE + 4, 0, 10, 4, 4, 1.0, 0, qc.QC_U8, FAKE, None) == 4
