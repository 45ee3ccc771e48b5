"""Pins of the workload tables (no GPU): the paper's own printed numbers fix the
ResNet-50 layer list and order that configs C3/C5 and the bench use."""
import os

import numpy as np

from workloads import (C1, RESNET50_LAYERS, S4, S8, U4, U8, make_layer_inputs, pack_codes,
                       resnet50_convs, resnet50_unique, unpack_codes, vgg16_convs)

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "fig13_im2col_overhead.txt")


def _read_golden():
    vals = {}
    for line in open(GOLDEN):
        if line.startswith("#") or not line.strip():
            continue
        parts = line.split()
        vals[parts[0]] = (float(parts[1]), parts[2] if len(parts) > 2 else None)
    return vals


def test_fig13_im2col_overhead_reproduces_paper():
    """min 1.0218x (conv18), max 8.6034x (conv2), avg 1.9445x."""
    g = _read_golden()
    over = []
    for cs in resnet50_unique(1):
        inp = cs.h * cs.w * cs.c
        col = cs.p * cs.q * cs.r * cs.s * cs.c
        wts = cs.k * cs.r * cs.s * cs.c
        over.append((inp + col + wts) / (inp + wts))
    assert len(over) == 19
    i_min, i_max = int(np.argmin(over)), int(np.argmax(over))
    assert round(over[i_min], 4) == g["min"][0] and f"conv{i_min + 1}" == g["min"][1]
    assert round(over[i_max], 4) == g["max"][0] and f"conv{i_max + 1}" == g["max"][1]
    assert round(float(np.mean(over)), 4) == g["avg"][0]


def test_resnet50_table():
    L = resnet50_convs(32)
    assert len(L) == 53
    # conv1 and conv3 are 1x1 kernels with 64 input channels
    u = resnet50_unique(1)
    assert (u[0].r, u[0].c) == (1, 64) and (u[2].r, u[2].c) == (1, 64)
    gmac = sum(cs.macs for cs in L) / 32
    assert abs(2 * gmac / 1e9 - 7.71) < 0.01          # 7.71 GOP per image
    assert RESNET50_LAYERS[0]["role"] == "stem"
    assert len(vgg16_convs(64)) == 13
    assert (C1.p, C1.q) == (56, 56)


def test_pack_roundtrip_and_nibble_order():
    rng = np.random.default_rng(0)
    for t, lo, hi in [(U4, 0, 15), (S4, -8, 7), (U8, 0, 255), (S8, -128, 127)]:
        codes = rng.integers(lo, hi + 1, size=(3, 5, 8))
        np.testing.assert_array_equal(unpack_codes(pack_codes(codes, t), t, 8), codes)
    assert pack_codes(np.array([[1, 2]]), U4)[0, 0] == 0x21
    assert pack_codes(np.array([[-1, 1]]), S4)[0, 0] == 0x1F


def test_generators_are_seeded():
    a = make_layer_inputs(C1, 8, seed=5)
    b = make_layer_inputs(C1, 8, seed=5)
    np.testing.assert_array_equal(a.x_bytes, b.x_bytes)
    np.testing.assert_array_equal(a.w_bytes, b.w_bytes)
    assert a.x_t == U8 and a.w_t == S8
    # post-ReLU recipe: about half zeros
    assert 0.4 < float(np.mean(a.x_codes == 0)) < 0.65
