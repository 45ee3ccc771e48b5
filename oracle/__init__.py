"""CPU oracle for the quantized-convolution hot path -- TEST INFRASTRUCTURE.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
`--impl reference` legs may import this package.  The product path
(paper_conf_icpp_hanhyylhgwwlq20_b200) never imports it, and it imports
nothing from the product path: the two share no code.

The arithmetic lives in oracle.c (plain C, int64/int128, OpenMP over (n,p)),
each function citing the passage of /root/reference/PAPER.md it follows; this
module is only ctypes marshalling.  Parity status of every function is pinned
(see tests/test_oracle_pins.py and DESIGN.md section 3); nothing here is
"parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")

U4, S4, U8, S8, S32, F32, BF16 = 0, 1, 2, 3, 4, 5, 6
_BITS = {U4: 4, S4: 4, U8: 8, S8: 8, S32: 32, F32: 32, BF16: 16}
ROUND_SINGLE, ROUND_TFLITE = 0, 1


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so (gcc, OpenMP, no fast-math)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=gnu11", "-fno-fast-math",
               "-ffp-contract=off", "-o", _SO, _SRC, "-lm"]
        subprocess.check_call(cmd)
    return _SO


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        vp, i32, i64, f32 = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_float
        L.oracle_quantize.argtypes = [vp, i32, i64, i32, i32, f32, i32, i32, vp]
        L.oracle_quantize.restype = i32
        L.oracle_requant_params.argtypes = [f32, vp, f32, i32, vp, vp]
        L.oracle_requant_params.restype = i32
        L.oracle_conv2d.argtypes = [i32] * 7 + [i32] * 6 + [i32] * 3 + [i32, vp, i32, i32, i32] \
            + [vp, vp, vp, vp, vp, vp]
        L.oracle_conv2d.restype = i64
        L.oracle_conv2d_ex.argtypes = [i32] * 7 + [i32] * 6 + [i32] * 3 + [i32, vp, i32, i32, i32, i32] \
            + [vp, vp, vp, vp, vp, vp, i32, vp]
        L.oracle_conv2d_ex.restype = i64
        L.oracle_srdhm.argtypes = [ctypes.c_int32, ctypes.c_int32]
        L.oracle_srdhm.restype = ctypes.c_int32
        L.oracle_rdbpot.argtypes = [ctypes.c_int32, i32]
        L.oracle_rdbpot.restype = ctypes.c_int32
        _lib = L
    return _lib


def _ptr(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def quantize(x: np.ndarray, scale: float, zero_point: int, yt: int, c_pad: Optional[int] = None,
             bf16: bool = False) -> np.ndarray:
    """x: fp32 [..., C] (or uint16 bf16 bit patterns with bf16=True) -> packed uint8
    [..., C_pad*bits/8].  Follows oracle.c:oracle_quantize (reading Z4)."""
    x = np.ascontiguousarray(x, dtype=np.uint16 if bf16 else np.float32)
    c = x.shape[-1]
    c_pad = c if c_pad is None else c_pad
    npix = int(np.prod(x.shape[:-1]))
    nbytes = c_pad * _BITS[yt] // 8
    y = np.zeros(x.shape[:-1] + (nbytes,), dtype=np.uint8)
    rc = lib().oracle_quantize(_ptr(x), 1 if bf16 else 0, npix, c, c_pad, float(scale),
                               int(zero_point), int(yt), _ptr(y))
    if rc != 0:
        raise ValueError("oracle_quantize: invalid arguments")
    return y


def requant_params(in_scale: float, w_scale: np.ndarray, out_scale: float):
    """Reading R1 -> (multiplier int32[K], shift int32[K])."""
    ws = np.ascontiguousarray(w_scale, dtype=np.float32)
    k = ws.shape[0]
    m = np.zeros(k, dtype=np.int32)
    n = np.zeros(k, dtype=np.int32)
    rc = lib().oracle_requant_params(float(in_scale), _ptr(ws), float(out_scale), k, _ptr(m), _ptr(n))
    if rc != 0:
        raise ValueError("oracle_requant_params: invalid arguments")
    return m, n


def conv_out_hw(h, w, r, s, stride_h, stride_w, pad_h, pad_w, dil_h, dil_w):
    p = (h + 2 * pad_h - dil_h * (r - 1) - 1) // stride_h + 1
    q = (w + 2 * pad_w - dil_w * (s - 1) - 1) // stride_w + 1
    return p, q


def conv2d(x: np.ndarray, w: np.ndarray, *, n, h, wd, c, k, r, s, xt, wt, yt,
           stride=(1, 1), pad=(0, 0), dil=(1, 1), x_zero=0, w_zero=None, y_zero=0,
           clamp_lo=None, clamp_hi=None, bias=None, mult=None, shift=None,
           rounding=ROUND_SINGLE, dq_scale=None, relu=False,
           allow_overflow=False) -> np.ndarray:
    """Direct 7-loop quantized convolution (oracle.c:oracle_conv2d_ex).

    x, w: packed uint8 buffers (NHWC / KRSC).  Returns the packed output
    buffer [n, p, q, k*bits/8] (uint8), int32 [n,p,q,k] for yt == S32, float32
    [n,p,q,k] for yt == F32 and uint16 bf16 bit patterns [n,p,q,k] for BF16."""
    p, q = conv_out_hw(h, wd, r, s, stride[0], stride[1], pad[0], pad[1], dil[0], dil[1])
    x = np.ascontiguousarray(x, dtype=np.uint8)
    w = np.ascontiguousarray(w, dtype=np.uint8)
    if clamp_lo is None or clamp_hi is None:
        lo = {U4: 0, S4: -8, U8: 0, S8: -128}.get(yt, 0)
        hi = {U4: 15, S4: 7, U8: 255, S8: 127}.get(yt, 0)
        clamp_lo = lo if clamp_lo is None else clamp_lo
        clamp_hi = hi if clamp_hi is None else clamp_hi
    bias = None if bias is None else np.ascontiguousarray(bias, dtype=np.int32)
    mult = None if mult is None else np.ascontiguousarray(mult, dtype=np.int32)
    shift = None if shift is None else np.ascontiguousarray(shift, dtype=np.int32)
    dqs = None if dq_scale is None else np.ascontiguousarray(dq_scale, dtype=np.float32)
    wz = None if w_zero is None else np.ascontiguousarray(w_zero, dtype=np.int32)
    if yt == S32:
        y = np.zeros((n, p, q, k), dtype=np.int32)
    elif yt == F32:
        y = np.zeros((n, p, q, k), dtype=np.float32)
    elif yt == BF16:
        y = np.zeros((n, p, q, k), dtype=np.uint16)
    else:
        y = np.zeros((n, p, q, k * _BITS[yt] // 8), dtype=np.uint8)
    ov = lib().oracle_conv2d_ex(n, h, wd, c, k, r, s, stride[0], stride[1], pad[0], pad[1],
                                dil[0], dil[1], xt, wt, yt, int(x_zero), _ptr(wz), int(y_zero),
                                int(clamp_lo), int(clamp_hi), int(rounding), _ptr(x), _ptr(w),
                                _ptr(bias), _ptr(mult), _ptr(shift), _ptr(dqs), int(bool(relu)),
                                _ptr(y))
    if ov < 0:
        raise ValueError("oracle_conv2d_ex: invalid arguments")
    if ov > 0 and not allow_overflow:
        raise OverflowError(f"oracle_conv2d: {ov} accumulators outside int32 (outside the contract)")
    return y


def srdhm(a: int, b: int) -> int:
    """gemmlowp SaturatingRoundingDoublingHighMul (oracle.c, reading Z15)."""
    return int(lib().oracle_srdhm(int(a), int(b)))


def rdbpot(x: int, e: int) -> int:
    """gemmlowp RoundingDivideByPOT (oracle.c, reading Z15)."""
    return int(lib().oracle_rdbpot(int(x), int(e)))


def conv2d_layer(li, mult=None, shift=None, y_t=None, bias=True, n_slice=None, **kw):
    """Convenience: run the oracle on a workloads.LayerInputs (optionally a batch slice);
    extra keywords (rounding, dq_scale, relu, w_zero, ...) go to conv2d."""
    cs = li.shape
    yt = li.y_t if y_t is None else y_t
    c_st = li.x_codes.shape[-1]
    xb = li.x_bytes
    n = cs.n
    if n_slice is not None:
        xb = xb[n_slice]
        n = xb.shape[0]
    return conv2d(xb, li.w_bytes, n=n, h=cs.h, wd=cs.w, c=c_st, k=cs.k, r=cs.r, s=cs.s,
                  xt=li.x_t, wt=li.w_t, yt=yt, stride=(cs.stride, cs.stride),
                  pad=(cs.pad, cs.pad), dil=(cs.dil, cs.dil), x_zero=li.x_zero, y_zero=li.y_zero,
                  clamp_lo=li.clamp_lo, clamp_hi=li.clamp_hi,
                  bias=li.bias if bias else None, mult=mult, shift=shift, **kw)
