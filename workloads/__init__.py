"""Seeded synthetic workloads (shapes + input generators) shared by tests and bench.

This module holds NO arithmetic of the method: it only states layer shapes
(the paper's ResNet-50 layer list, VGG-16, BASELINE.json configs) and draws
seeded random inputs with the value distributions of the paper's workloads
(recipe restated in DESIGN.md section 5).  It packs
integer codes into the byte layout the boundary consumes (NHWC activations,
KRSC weights, 4-bit element 2j in the low nibble of byte j -- reading Z7).
Re-quantization multipliers are NOT derived here: consumers call either the
oracle (tests) or the library (bench) on the float scales drawn here.

Paper citations (P:Lnnn = /root/reference/PAPER.md line):
  * ResNet-50 "adopted from Caffe Model Zoo", all conv layers;
    19 unique non-stem shapes conv1..conv19 in network order; the order and
    shapes are pinned by Fig.13's im2col overhead in
    tests/test_workloads.py and by "conv1 and conv3 ... 1x1 kernel with 64
    channels".
  * NHWC layout on GPU.
"""
from __future__ import annotations

import dataclasses
from typing import Dict, List, Optional

import numpy as np

# dtype codes of the boundary (include/qconv.h qc_dtype); plain ints, no logic.
U4, S4, U8, S8, S32 = 0, 1, 2, 3, 4
DTYPE_NAMES = {U4: "u4", S4: "s4", U8: "u8", S8: "s8", S32: "s32"}
DTYPE_RANGE = {U4: (0, 15), S4: (-8, 7), U8: (0, 255), S8: (-128, 127),
               S32: (-(2 ** 31), 2 ** 31 - 1)}
DTYPE_BITS = {U4: 4, S4: 4, U8: 8, S8: 8, S32: 32}

SEED_BASE = 20200817


@dataclasses.dataclass(frozen=True)
class ConvShape:
    name: str
    n: int
    h: int
    w: int
    c: int
    k: int
    r: int
    s: int
    stride: int = 1
    pad: int = 0
    dil: int = 1

    @property
    def p(self) -> int:
        return (self.h + 2 * self.pad - self.dil * (self.r - 1) - 1) // self.stride + 1

    @property
    def q(self) -> int:
        return (self.w + 2 * self.pad - self.dil * (self.s - 1) - 1) // self.stride + 1

    @property
    def macs(self) -> int:
        return self.n * self.p * self.q * self.k * self.r * self.s * self.c

    def with_batch(self, n: int) -> "ConvShape":
        return dataclasses.replace(self, n=n)


def _resnet50_layers() -> List[dict]:
    """53 conv layers of Caffe ResNet-50 (stride on the 1x1 branch2a/branch1),
    in network order, per image (n filled in by callers)."""
    L = [dict(name="conv1", h=224, w=224, c=3, k=64, r=7, s=7, stride=2, pad=3, role="stem")]
    stages = [("res2", 3, 64, 56, 1), ("res3", 4, 128, 56, 2), ("res4", 6, 256, 28, 2),
              ("res5", 3, 512, 14, 2)]
    cin = 64
    for sname, nblocks, width, hin, first_stride in stages:
        h = hin
        for b in range(nblocks):
            blk = f"{sname}{chr(ord('a') + b)}"
            st = first_stride if b == 0 else 1
            ho = (h - 1) // st + 1
            L.append(dict(name=f"{blk}_branch2a", h=h, w=h, c=cin, k=width, r=1, s=1,
                          stride=st, pad=0, role="2a"))
            L.append(dict(name=f"{blk}_branch2b", h=ho, w=ho, c=width, k=width, r=3, s=3,
                          stride=1, pad=1, role="2b"))
            L.append(dict(name=f"{blk}_branch2c", h=ho, w=ho, c=width, k=4 * width, r=1, s=1,
                          stride=1, pad=0, role="2c"))
            if b == 0:
                L.append(dict(name=f"{blk}_branch1", h=h, w=h, c=cin, k=4 * width, r=1, s=1,
                              stride=st, pad=0, role="branch1"))
            cin = 4 * width
            h = ho
    return L


RESNET50_LAYERS: List[dict] = _resnet50_layers()


def resnet50_convs(batch: int) -> List[ConvShape]:
    return [ConvShape(name=d["name"], n=batch, h=d["h"], w=d["w"], c=d["c"], k=d["k"],
                      r=d["r"], s=d["s"], stride=d["stride"], pad=d["pad"])
            for d in RESNET50_LAYERS]


def resnet50_unique(batch: int = 1) -> List[ConvShape]:
    """The paper's conv1..conv19 (unique non-stem shapes, first-occurrence order)."""
    seen, out = set(), []
    for cs in resnet50_convs(batch)[1:]:
        key = (cs.h, cs.w, cs.c, cs.k, cs.r, cs.s, cs.stride, cs.pad)
        if key not in seen:
            seen.add(key)
            out.append(dataclasses.replace(cs, name=f"conv{len(out) + 1}:{cs.name}"))
    return out


def vgg16_convs(batch: int) -> List[ConvShape]:
    cfg = [(224, 3, 64), (224, 64, 64), (112, 64, 128), (112, 128, 128),
           (56, 128, 256), (56, 256, 256), (56, 256, 256),
           (28, 256, 512), (28, 512, 512), (28, 512, 512),
           (14, 512, 512), (14, 512, 512), (14, 512, 512)]
    names = ["conv1_1", "conv1_2", "conv2_1", "conv2_2", "conv3_1", "conv3_2", "conv3_3",
             "conv4_1", "conv4_2", "conv4_3", "conv5_1", "conv5_2", "conv5_3"]
    return [ConvShape(name=nm, n=batch, h=h, w=h, c=c, k=k, r=3, s=3, stride=1, pad=1)
            for nm, (h, c, k) in zip(names, cfg)]


# BASELINE.json configs[0..1]
C1 = ConvShape("C1_resnet18_conv2x", n=1, h=56, w=56, c=64, k=64, r=3, s=3, stride=1, pad=1)


def layer_role(name: str) -> str:
    for d in RESNET50_LAYERS:
        if d["name"] == name:
            return d["role"]
    return "2b"


# ---------------------------------------------------------------------------
# packing of integer codes into the boundary's byte layout (input encoding)

def pack_codes(codes: np.ndarray, dtype: int) -> np.ndarray:
    """int array [..., C] -> uint8 bytes [..., C*bits/8] (row-major; Z7 nibble order)."""
    codes = np.asarray(codes)
    lo, hi = DTYPE_RANGE[dtype]
    assert codes.min(initial=lo) >= lo and codes.max(initial=hi) <= hi, "code out of range"
    if dtype == S32:
        return codes.astype("<i4").view(np.uint8).reshape(*codes.shape[:-1], -1)
    if DTYPE_BITS[dtype] == 8:
        return (codes.astype(np.int64) & 0xFF).astype(np.uint8)
    assert codes.shape[-1] % 2 == 0, "4-bit rows need an even element count"
    u = (codes.astype(np.int64) & 0xF).astype(np.uint8)
    return (u[..., 0::2] | (u[..., 1::2] << 4)).astype(np.uint8)


def unpack_codes(buf: np.ndarray, dtype: int, count: int) -> np.ndarray:
    """Inverse of pack_codes along the last axis (count elements per row)."""
    buf = np.asarray(buf, dtype=np.uint8)
    if dtype == S32:
        return np.ascontiguousarray(buf).view("<i4").astype(np.int64)
    if DTYPE_BITS[dtype] == 8:
        return buf.astype(np.int8 if dtype == S8 else np.uint8).astype(np.int64)
    lo = (buf & 0xF).astype(np.int64)
    hi = (buf >> 4).astype(np.int64)
    out = np.empty(buf.shape[:-1] + (buf.shape[-1] * 2,), dtype=np.int64)
    out[..., 0::2], out[..., 1::2] = lo, hi
    if dtype == S4:
        out = np.where(out >= 8, out - 16, out)
    return out[..., :count]


# ---------------------------------------------------------------------------
# seeded generators (recipe: DESIGN.md section 5 / SURVEY.md 8(d))

@dataclasses.dataclass
class LayerInputs:
    shape: ConvShape
    x_t: int
    w_t: int
    y_t: int
    x_codes: np.ndarray      # int64 [N,H,W,C]
    w_codes: np.ndarray      # int64 [K,R,S,C]
    x_bytes: np.ndarray      # uint8 packed NHWC
    w_bytes: np.ndarray      # uint8 packed KRSC
    bias: np.ndarray         # int32 [K]
    x_zero: int
    y_zero: int
    clamp_lo: int
    clamp_hi: int
    s_x: float
    s_w: np.ndarray          # float32 [K]
    s_y: float
    relu: bool


def post_relu_codes(rng: np.random.Generator, shape, bits: int, sigma_frac: float = 40 / 255):
    """Half-normal "post-ReLU" activation codes: ~50% zeros, rest round(|N(0, sigma)|)."""
    qmax = (1 << bits) - 1
    v = np.rint(np.abs(rng.normal(0.0, sigma_frac * qmax, size=shape)))
    v = np.where(rng.random(shape) < 0.5, 0.0, v)
    return np.clip(v, 0, qmax).astype(np.int64)


def symmetric_weight_codes(rng: np.random.Generator, k: int, rsc: tuple, bits: int):
    """Per-output-channel symmetric weights round(N(0,1) * qmax / max|w_k|)."""
    qmax = (1 << (bits - 1)) - 1
    wf = rng.normal(0.0, 1.0, size=(k,) + rsc)
    amax = np.abs(wf.reshape(k, -1)).max(axis=1)
    amax = np.where(amax == 0, 1.0, amax)
    codes = np.rint(wf / amax.reshape((k,) + (1,) * len(rsc)) * qmax).astype(np.int64)
    return codes, (amax / qmax).astype(np.float32)


def make_layer_inputs(cs: ConvShape, bits: int, seed: int, *, out_bits: Optional[int] = None,
                      signed_out: bool = False, relu: bool = True, x_zero: int = 0,
                      uniform_x: bool = False, c_store: Optional[int] = None) -> LayerInputs:
    """Draw one layer's inputs.  `c_store` pads the stored channel count (the
    extra channels hold x_zero codes and zero weights, so the conv result is
    unchanged -- used for the C=3 stem)."""
    rng = np.random.default_rng(seed)
    out_bits = bits if out_bits is None else out_bits
    x_t = U4 if bits == 4 else U8
    w_t = S4 if bits == 4 else S8
    if out_bits == 32:
        y_t = S32
    elif out_bits == 4:
        y_t = S4 if signed_out else U4
    else:
        y_t = S8 if signed_out else U8
    c_st = cs.c if c_store is None else c_store
    qx_max = (1 << bits) - 1
    if uniform_x:
        x_codes = rng.integers(0, qx_max + 1, size=(cs.n, cs.h, cs.w, cs.c)).astype(np.int64)
    else:
        x_codes = post_relu_codes(rng, (cs.n, cs.h, cs.w, cs.c), bits)
    if x_zero:
        x_codes = np.clip(x_codes + x_zero - (qx_max + 1) // 4, 0, qx_max)
    w_codes, s_w = symmetric_weight_codes(rng, cs.k, (cs.r, cs.s, cs.c), bits)
    bias = rng.integers(-(1 << 12), (1 << 12) + 1, size=cs.k).astype(np.int32)
    if c_st != cs.c:
        xp = np.full((cs.n, cs.h, cs.w, c_st), x_zero, dtype=np.int64)
        xp[..., :cs.c] = x_codes
        wp = np.zeros((cs.k, cs.r, cs.s, c_st), dtype=np.int64)
        wp[..., :cs.c] = w_codes
        x_codes, w_codes = xp, wp
    s_x = np.float32(0.05)
    # output scale: ~1% of post-ReLU outputs clip at qmax (analytic estimate
    # from the code statistics; a recipe, not part of the method)
    xc = (x_codes - x_zero).astype(np.float64)
    ex2 = float(np.mean(xc ** 2)) if xc.size else 1.0
    ew2 = float(np.mean(w_codes.astype(np.float64) ** 2))
    sigma_acc = np.sqrt(cs.r * cs.s * cs.c * ex2 * ew2) + 1.0
    if y_t == S32:
        qy_max = 1
    else:
        qy_max = DTYPE_RANGE[y_t][1]
    s_w_med = float(np.median(s_w))
    s_y = np.float32(float(s_x) * s_w_med * 2.33 * sigma_acc / max(qy_max, 1))
    y_zero = 0
    lo, hi = DTYPE_RANGE[y_t] if y_t != S32 else (0, 0)
    if relu and y_t != S32:
        lo = max(lo, y_zero)
    return LayerInputs(shape=cs, x_t=x_t, w_t=w_t, y_t=y_t, x_codes=x_codes, w_codes=w_codes,
                       x_bytes=pack_codes(x_codes, x_t), w_bytes=pack_codes(w_codes, w_t),
                       bias=bias, x_zero=int(x_zero), y_zero=y_zero, clamp_lo=int(lo),
                       clamp_hi=int(hi), s_x=float(s_x), s_w=s_w, s_y=float(s_y), relu=relu)


@dataclasses.dataclass
class LayerParams:
    """Weights and scales of one layer (no activations) -- for the bench trunk."""
    shape: ConvShape
    x_t: int
    w_t: int
    y_t: int
    w_codes: np.ndarray
    w_bytes: np.ndarray
    bias: np.ndarray
    s_x: float
    s_w: np.ndarray
    s_y: float
    clamp_lo: int
    clamp_hi: int
    c_store: int


def make_layer_params(cs: ConvShape, bits: int, seed: int, *, c_store: Optional[int] = None,
                      relu: bool = True) -> LayerParams:
    """Seeded weights/bias/scales with the same recipe as make_layer_inputs; the output
    scale uses the expected second moment of post-ReLU half-normal activation codes."""
    rng = np.random.default_rng(seed)
    x_t = U4 if bits == 4 else U8
    w_t = S4 if bits == 4 else S8
    y_t = x_t
    c_st = cs.c if c_store is None else c_store
    w_codes, s_w = symmetric_weight_codes(rng, cs.k, (cs.r, cs.s, cs.c), bits)
    bias = rng.integers(-(1 << 12), (1 << 12) + 1, size=cs.k).astype(np.int32)
    if bits == 4:
        bias = (bias // 64).astype(np.int32)
    if c_st != cs.c:
        wp = np.zeros((cs.k, cs.r, cs.s, c_st), dtype=np.int64)
        wp[..., :cs.c] = w_codes
        w_codes = wp
    qx_max = (1 << bits) - 1
    sig = 40 / 255 * qx_max
    ex2 = 0.5 * sig * sig
    ew2 = float(np.mean(w_codes[..., :cs.c].astype(np.float64) ** 2))
    sigma_acc = np.sqrt(cs.r * cs.s * cs.c * ex2 * ew2) + 1.0
    s_x = np.float32(0.05)
    s_y = np.float32(float(s_x) * float(np.median(s_w)) * 2.33 * sigma_acc / DTYPE_RANGE[y_t][1])
    lo, hi = DTYPE_RANGE[y_t]
    packable = DTYPE_BITS[w_t] == 8 or w_codes.shape[-1] % 2 == 0
    return LayerParams(shape=cs, x_t=x_t, w_t=w_t, y_t=y_t, w_codes=w_codes,
                       w_bytes=pack_codes(w_codes, w_t) if packable else None, bias=bias, s_x=float(s_x), s_w=s_w,
                       s_y=float(s_y), clamp_lo=max(lo, 0) if relu else lo, clamp_hi=hi,
                       c_store=c_st)


def post_relu_codes_fast(rng: np.random.Generator, shape, bits: int) -> np.ndarray:
    """uint8 post-ReLU codes (same distribution as post_relu_codes, less memory)."""
    qmax = (1 << bits) - 1
    v = np.abs(rng.standard_normal(size=shape, dtype=np.float32)) * np.float32(40 / 255 * qmax)
    v = np.rint(v)
    v[rng.random(size=shape, dtype=np.float32) < 0.5] = 0
    return np.clip(v, 0, qmax).astype(np.uint8)


def stored_channels(cs: ConvShape, bits: int) -> int:
    """Stored channel count the library accepts for this layer (C padded to a
    multiple of 32 elements only where the real C is smaller, i.e. the stem)."""
    if cs.c % 32 == 0:
        return cs.c
    return ((cs.c + 31) // 32) * 32


def layer_seed(index: int) -> int:
    return SEED_BASE + index


def float_image(rng: np.random.Generator, shape) -> np.ndarray:
    """fp32 activations ReLU(N(0,1)) (C2 recipe)."""
    return np.maximum(rng.normal(0.0, 1.0, size=shape), 0.0).astype(np.float32)


def device_post_relu_codes(shape, bits: int, seed: int, device):
    """Packed post-ReLU activation codes drawn on the GPU with a seeded torch generator (same
    recipe as post_relu_codes: ~50 % zeros, rest round(|N(0, 40/255 * qmax)|) clipped) -- for
    bench-sized layers whose inputs are too large to draw on the host.  Returns a uint8 tensor
    [..., C * bits / 8] in the boundary's byte layout (Z7 nibble order)."""
    import torch
    g = torch.Generator(device=device)
    g.manual_seed(int(seed))
    qmax = (1 << bits) - 1
    v = torch.randn(shape, generator=g, device=device).abs_().mul_(40 / 255 * qmax).round_()
    v[torch.rand(shape, generator=g, device=device) < 0.5] = 0
    codes = v.clamp_(0, qmax).to(torch.uint8)
    if bits == 4:
        return (codes[..., 0::2] | (codes[..., 1::2] << 4)).contiguous()
    return codes


def densenet121_convs(batch: int) -> List[ConvShape]:
    """The 120 conv layers of DenseNet-121 (growth 32, bottleneck 4 x 32, blocks 6/12/24/16,
    compression 0.5) in network order -- the paper's second GPU workload (Fig.17:
    "input size for conv15 ... is 1 x 14 x 14 x 736").  The stem is 7x7/s2 over C = 3."""
    out = [ConvShape("dn_conv0", batch, 224, 224, 3, 64, 7, 7, 2, 3)]
    c, hw = 64, 56
    for b, nl in enumerate((6, 12, 24, 16)):
        for i in range(nl):
            cin = c + 32 * i
            out.append(ConvShape(f"dn_b{b + 1}_l{i + 1}_1x1", batch, hw, hw, cin, 128, 1, 1))
            out.append(ConvShape(f"dn_b{b + 1}_l{i + 1}_3x3", batch, hw, hw, 128, 32, 3, 3, 1, 1))
        c += 32 * nl
        if b < 3:
            out.append(ConvShape(f"dn_t{b + 1}", batch, hw, hw, c, c // 2, 1, 1))
            c //= 2
            hw //= 2
    return out


def densenet121_unique(batch: int = 1) -> List[ConvShape]:
    """Unique DenseNet-121 conv shapes (first occurrence order), stem excluded."""
    seen, out = set(), []
    for cs in densenet121_convs(batch)[1:]:
        key = (cs.h, cs.w, cs.c, cs.k, cs.r, cs.s, cs.stride, cs.pad)
        if key not in seen:
            seen.add(key)
            out.append(cs)
    return out
