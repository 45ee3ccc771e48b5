"""B200-native 4/8-bit quantized convolution (Han, Hu et al., ICPP'20, section 4).

Thin Python binding over the C ABI of libqconv.so (include/qconv.h): argument
marshalling only -- every step of the hot path (quantize+pack, implicit-GEMM
convolution on tcgen05 tensor cores, fused bias/re-quantization/ReLU/packing)
runs in the library's CUDA kernels.  PyTorch is used for device memory and
streams.  There is no CPU fallback: if libqconv.so is missing, importing
this package raises.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass
from typing import Optional, Sequence, Tuple

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_PKG, "libqconv.so")

QC_U4, QC_S4, QC_U8, QC_S8, QC_S32, QC_F32_OUT, QC_BF16_OUT = 0, 1, 2, 3, 4, 5, 6
QC_F32, QC_BF16 = 0, 1
QC_ROUND_SINGLE, QC_ROUND_TFLITE = 0, 1
QC_KERNEL_AUTO, QC_KERNEL_IM2COL, QC_KERNEL_PAIR, QC_KERNEL_HALO, QC_KERNEL_CHANNEL, QC_KERNEL_HALO_T = 0, 1, 2, 3, 4, 5
KERNEL_NAMES = {0: "auto", 1: "im2col", 2: "pair", 3: "halo", 4: "channel", 5: "halo_t"}
_BITS = {QC_U4: 4, QC_S4: 4, QC_U8: 8, QC_S8: 8, QC_S32: 32, QC_F32_OUT: 32, QC_BF16_OUT: 16}
_RANGE = {QC_U4: (0, 15), QC_S4: (-8, 7), QC_U8: (0, 255), QC_S8: (-128, 127),
          QC_S32: (-(2 ** 31), 2 ** 31 - 1)}

STATUS = {0: "QC_OK", 1: "QC_ERR_INVALID_ARG", 2: "QC_ERR_UNSUPPORTED", 3: "QC_ERR_OVERFLOW_RISK",
          4: "QC_ERR_MISALIGNED", 5: "QC_ERR_WORKSPACE", 6: "QC_ERR_CUDA"}


class QConvError(RuntimeError):
    def __init__(self, fn: str, status: int, cuda_err: int = 0):
        self.status = status
        msg = f"{fn}: {STATUS.get(status, status)} ({_lib().qconv_status_string(status).decode()})"
        if status == 6:
            msg += f" cudaError={cuda_err}"
        super().__init__(msg)


class qconv_desc(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in
                ("n", "h", "w", "c", "k", "r", "s", "stride_h", "stride_w", "pad_h", "pad_w",
                 "dil_h", "dil_w", "x_t", "w_t", "y_t", "x_zero")] + \
               [("w_zero", ctypes.c_void_p)] + \
               [(n, ctypes.c_int32) for n in ("w_prepared", "y_zero", "clamp_lo", "clamp_hi",
                                               "rounding", "relu")]


class qconv_plan(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in
                ("kernel", "bn", "bm", "stages", "grid", "threads", "num_tiles", "smem_bytes",
                 "tmem_cols", "prologue", "epilogue_mode")] + [("reserved", ctypes.c_int32 * 5)]

    def as_dict(self):
        d = {f: getattr(self, f) for f, _ in self._fields_ if f != "reserved"}
        d["kernel_name"] = KERNEL_NAMES.get(self.kernel, str(self.kernel))
        return d


_L = None


def _lib():
    global _L
    if _L is None:
        if not os.path.exists(_SO):
            raise ImportError(f"libqconv.so not built at {_SO}; run __graft_entry__.build() "
                              "(no CPU fallback exists)")
        L = ctypes.CDLL(_SO)
        vp, i32, i64, f32, sz = (ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_float,
                                 ctypes.c_size_t)
        dp = ctypes.POINTER(qconv_desc)
        L.qconv_status_string.argtypes = [i32]
        L.qconv_status_string.restype = ctypes.c_char_p
        L.qconv_last_cuda_error.restype = i32
        L.qconv_version.restype = i32
        L.qconv_quantize_pack.argtypes = [vp, i32, i64, i32, i32, f32, i32, i32, vp, vp]
        L.qconv_quantize_pack.restype = i32
        L.qconv_requant_params.argtypes = [f32, vp, f32, i32, vp, vp]
        L.qconv_requant_params.restype = i32
        L.qconv_prepared_weight_bytes.argtypes = [dp]
        L.qconv_prepared_weight_bytes.restype = sz
        L.qconv_prepare_weights.argtypes = [dp, vp, vp, vp]
        L.qconv_prepare_weights.restype = i32
        L.qconv2d_workspace_size.argtypes = [dp]
        L.qconv2d_workspace_size.restype = sz
        L.qconv2d_forward.argtypes = [dp, vp, vp, vp, vp, vp, vp, vp, sz, vp]
        L.qconv2d_forward.restype = i32
        L.qconv2d_forward_dequant.argtypes = [dp, vp, vp, vp, vp, vp, vp, sz, vp]
        L.qconv2d_forward_dequant.restype = i32
        L.qconv2d_quantize_workspace_size.argtypes = [dp, i32]
        L.qconv2d_quantize_workspace_size.restype = sz
        L.qconv2d_forward_quantize.argtypes = [dp, vp, i32, f32, vp, vp, vp, vp, vp, vp, sz, vp]
        L.qconv2d_forward_quantize.restype = i32
        pp = ctypes.POINTER(qconv_plan)
        L.qconv_debug_plan.argtypes = [dp, pp]
        L.qconv_debug_plan.restype = i32
        L.qconv_debug_plan_quantize.argtypes = [dp, i32, pp]
        L.qconv_debug_plan_quantize.restype = i32
        L.qconv_plan_set.argtypes = [dp, pp]
        L.qconv_plan_set.restype = i32
        L.qconv_plan_clear.argtypes = []
        L.qconv_plan_clear.restype = None
        L.qconv_plan_candidates.argtypes = [dp, pp, i32]
        L.qconv_plan_candidates.restype = i32
        L.qconv_autotune.argtypes = [dp, vp, vp, vp, vp, vp, vp, vp, sz, vp, i32, pp,
                                     ctypes.POINTER(ctypes.c_float)]
        L.qconv_autotune.restype = i32
        L.qconv_s2d_desc.argtypes = [dp, dp]
        L.qconv_s2d_desc.restype = i32
        L.qconv_quantize_pack_s2d.argtypes = [dp, vp, i32, f32, vp, vp]
        L.qconv_quantize_pack_s2d.restype = i32
        L.qconv_prepared_weight_bytes_s2d.argtypes = [dp]
        L.qconv_prepared_weight_bytes_s2d.restype = sz
        L.qconv_prepare_weights_s2d.argtypes = [dp, vp, vp, vp]
        L.qconv_prepare_weights_s2d.restype = i32
        L.qconv_debug_im2col_tile.argtypes = [dp, vp, i64, i32, i32, i32, i32, vp, vp]
        L.qconv_debug_im2col_tile.restype = i32
        _L = L
    return _L


def lib_path() -> str:
    return _SO


def _check(fn: str, st: int):
    if st != 0:
        raise QConvError(fn, st, _lib().qconv_last_cuda_error())


def _ptr(t) -> Optional[int]:
    if t is None:
        return None
    return t.data_ptr()


def _stream(stream) -> Optional[int]:
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream)


# --------------------------------------------------------------------------- descriptors
def make_desc(n, h, w, c, k, r, s, *, stride=1, pad=0, dil=1, x_t=QC_U8, w_t=QC_S8, y_t=QC_U8,
              x_zero=0, w_prepared=0, y_zero=0, clamp_lo=None, clamp_hi=None,
              relu=False, rounding=QC_ROUND_SINGLE, w_zero=None) -> qconv_desc:
    """Descriptor (include/qconv.h).  w_zero: optional device int32 tensor [k] of weight zero
    points -- the caller keeps it alive while the descriptor is used.  relu: for integer
    outputs it narrows clamp_lo to max(qmin, y_zero); for float outputs it sets the
    descriptor's relu flag."""
    sh, sw = (stride, stride) if isinstance(stride, int) else stride
    ph, pw = (pad, pad) if isinstance(pad, int) else pad
    dh, dw = (dil, dil) if isinstance(dil, int) else dil
    packed = y_t in (QC_U4, QC_S4, QC_U8, QC_S8)
    lo, hi = _RANGE[y_t] if packed else (0, 0)
    if relu and packed:
        lo = max(lo, y_zero)
    lo = lo if clamp_lo is None else clamp_lo
    hi = hi if clamp_hi is None else clamp_hi
    wz = None if w_zero is None else (w_zero if isinstance(w_zero, int) else w_zero.data_ptr())
    return qconv_desc(n, h, w, c, k, r, s, sh, sw, ph, pw, dh, dw, x_t, w_t, y_t, x_zero, wz,
                      w_prepared, y_zero, lo, hi, rounding, 1 if (relu and not packed) else 0)


def out_hw(d: qconv_desc) -> Tuple[int, int]:
    p = (d.h + 2 * d.pad_h - d.dil_h * (d.r - 1) - 1) // d.stride_h + 1
    q = (d.w + 2 * d.pad_w - d.dil_w * (d.s - 1) - 1) // d.stride_w + 1
    return p, q


def output_nbytes_per_pixel(d: qconv_desc) -> int:
    return d.k * _BITS[d.y_t] // 8


# --------------------------------------------------------------------------- the C ABI
def qconv_quantize_pack(x, scale: float, zero_point: int, yt: int, c_pad: Optional[int] = None,
                        out=None, stream=None):
    """x: CUDA tensor fp32/bf16 [..., C] -> uint8 [..., C_pad*bits/8] (include/qconv.h)."""
    import torch
    assert x.is_cuda and x.is_contiguous()
    xt = QC_BF16 if x.dtype == torch.bfloat16 else QC_F32
    assert x.dtype in (torch.float32, torch.bfloat16)
    c = x.shape[-1]
    c_pad = c if c_pad is None else c_pad
    npix = x.numel() // c
    nbytes = c_pad * _BITS[yt] // 8
    if out is None:
        out = torch.empty(tuple(x.shape[:-1]) + (nbytes,), dtype=torch.uint8, device=x.device)
    _check("qconv_quantize_pack", _lib().qconv_quantize_pack(
        _ptr(x), xt, npix, c, c_pad, float(scale), int(zero_point), int(yt), _ptr(out),
        _stream(stream)))
    return out


def qconv_requant_params(in_scale: float, w_scale, out_scale: float):
    """Host-only (reading R1) -> (multiplier int32[K], shift int32[K]) numpy arrays."""
    ws = np.ascontiguousarray(np.asarray(w_scale, dtype=np.float32))
    k = ws.shape[0]
    m = np.zeros(k, dtype=np.int32)
    n = np.zeros(k, dtype=np.int32)
    _check("qconv_requant_params", _lib().qconv_requant_params(
        float(in_scale), ws.ctypes.data, float(out_scale), k, m.ctypes.data, n.ctypes.data))
    return m, n


def qconv_prepared_weight_bytes(d: qconv_desc) -> int:
    return int(_lib().qconv_prepared_weight_bytes(ctypes.byref(d)))


def qconv_prepare_weights(d: qconv_desc, w, out=None, stream=None):
    import torch
    nb = qconv_prepared_weight_bytes(d)
    if nb == 0:
        raise QConvError("qconv_prepare_weights", 1)
    if out is None:
        out = torch.empty(nb, dtype=torch.uint8, device=w.device)
    _check("qconv_prepare_weights", _lib().qconv_prepare_weights(
        ctypes.byref(d), _ptr(w), _ptr(out), _stream(stream)))
    return out


def qconv2d_workspace_size(d: qconv_desc) -> int:
    return int(_lib().qconv2d_workspace_size(ctypes.byref(d)))


def qconv2d_forward(d: qconv_desc, x, w, bias=None, multiplier=None, shift=None, y=None,
                    workspace=None, stream=None):
    """y = requant(conv(x - x_zero, w - w_zero) + bias) on the GPU (include/qconv.h)."""
    if y is None:
        y = _out_tensor(d, x.device)
    workspace, ws_bytes = _workspace(d, workspace, x.device)
    _check("qconv2d_forward", _lib().qconv2d_forward(
        ctypes.byref(d), _ptr(x), _ptr(w), _ptr(bias), _ptr(multiplier), _ptr(shift), _ptr(y),
        _ptr(workspace), ws_bytes, _stream(stream)))
    return y


def _out_tensor(d: qconv_desc, device):
    import torch
    p, q = out_hw(d)
    if d.y_t == QC_S32:
        return torch.empty((d.n, p, q, d.k), dtype=torch.int32, device=device)
    if d.y_t == QC_F32_OUT:
        return torch.empty((d.n, p, q, d.k), dtype=torch.float32, device=device)
    if d.y_t == QC_BF16_OUT:
        return torch.empty((d.n, p, q, d.k), dtype=torch.bfloat16, device=device)
    return torch.empty((d.n, p, q, output_nbytes_per_pixel(d)), dtype=torch.uint8, device=device)


def _workspace(d: qconv_desc, workspace, device):
    import torch
    ws_need = qconv2d_workspace_size(d)
    if ws_need and workspace is None:
        workspace = torch.empty(ws_need, dtype=torch.uint8, device=device)
    ws_bytes = 0 if workspace is None else workspace.numel() * workspace.element_size()
    return workspace, ws_bytes


def qconv2d_forward_dequant(d: qconv_desc, x, w, bias=None, scale=None, y=None, workspace=None,
                            stream=None):
    """y = fl32(fl32(conv(x - x_zero, w - w_zero) + bias) * scale[k]) (include/qconv.h),
    fp32 or bf16 per d.y_t."""
    if y is None:
        y = _out_tensor(d, x.device)
    workspace, ws_bytes = _workspace(d, workspace, x.device)
    _check("qconv2d_forward_dequant", _lib().qconv2d_forward_dequant(
        ctypes.byref(d), _ptr(x), _ptr(w), _ptr(bias), _ptr(scale), _ptr(y), _ptr(workspace),
        ws_bytes, _stream(stream)))
    return y


def qconv2d_forward_quantize(d: qconv_desc, x, in_scale: float, w, bias=None, multiplier=None,
                             shift=None, y=None, workspace=None, stream=None):
    """Float activations in: quantize (Z4, d.x_zero, d.x_t range) fused with the convolution
    (include/qconv.h); the C = 3 image stem runs as one kernel."""
    import torch
    assert x.is_cuda and x.is_contiguous() and x.dtype in (torch.float32, torch.bfloat16)
    xt = QC_BF16 if x.dtype == torch.bfloat16 else QC_F32
    if y is None:
        y = _out_tensor(d, x.device)
    need = int(_lib().qconv2d_quantize_workspace_size(ctypes.byref(d), xt))
    if need and workspace is None:
        workspace = torch.empty(need, dtype=torch.uint8, device=x.device)
    ws_bytes = 0 if workspace is None else workspace.numel() * workspace.element_size()
    _check("qconv2d_forward_quantize", _lib().qconv2d_forward_quantize(
        ctypes.byref(d), _ptr(x), xt, float(in_scale), _ptr(w), _ptr(bias), _ptr(multiplier),
        _ptr(shift), _ptr(y), _ptr(workspace), ws_bytes, _stream(stream)))
    return y


def qconv_debug_plan(d: qconv_desc) -> dict:
    """The launch plan qconv2d_forward would use for `d` (kernel family, tiles, grid, ...)."""
    p = qconv_plan()
    _check("qconv_debug_plan", _lib().qconv_debug_plan(ctypes.byref(d), ctypes.byref(p)))
    return p.as_dict()


def qconv_debug_plan_quantize(d: qconv_desc, xt: int = QC_F32) -> dict:
    """The launch plan of qconv2d_forward_quantize for `d` (float activations of type xt)."""
    p = qconv_plan()
    _check("qconv_debug_plan_quantize", _lib().qconv_debug_plan_quantize(ctypes.byref(d), int(xt),
                                                                         ctypes.byref(p)))
    return p.as_dict()


def qconv_plan_candidates(d: qconv_desc) -> list:
    n = _lib().qconv_plan_candidates(ctypes.byref(d), None, 0)
    arr = (qconv_plan * max(n, 1))()
    _lib().qconv_plan_candidates(ctypes.byref(d), arr, n)
    return [arr[i].as_dict() for i in range(n)]


def qconv_plan_set(d: qconv_desc, kernel: Optional[int] = None, bn: int = 0):
    """Record a (kernel, bn) choice for descriptors equal to `d`; kernel=None removes it."""
    if kernel is None:
        _check("qconv_plan_set", _lib().qconv_plan_set(ctypes.byref(d), None))
        return
    p = qconv_plan()
    p.kernel, p.bn = int(kernel), int(bn)
    _check("qconv_plan_set", _lib().qconv_plan_set(ctypes.byref(d), ctypes.byref(p)))


def qconv_plan_clear():
    _lib().qconv_plan_clear()


def qconv_autotune(d: qconv_desc, x, w, bias=None, multiplier=None, shift=None, y=None,
                   workspace=None, stream=None, iters: int = 10):
    """Profile-run search over the eligible plans; records and returns the best
    plan and its mean time in microseconds.  Synchronous."""
    if y is None:
        y = _out_tensor(d, x.device)
    workspace, ws_bytes = _workspace(d, workspace, x.device)
    best = qconv_plan()
    us = ctypes.c_float()
    _check("qconv_autotune", _lib().qconv_autotune(
        ctypes.byref(d), _ptr(x), _ptr(w), _ptr(bias), _ptr(multiplier), _ptr(shift), _ptr(y),
        _ptr(workspace), ws_bytes, _stream(stream), int(iters), ctypes.byref(best),
        ctypes.byref(us)))
    return best.as_dict(), float(us.value)


def qconv_s2d_desc(d: qconv_desc) -> qconv_desc:
    """Descriptor of the space-to-depth form of a stride-2 conv (include/qconv.h)."""
    o = qconv_desc()
    _check("qconv_s2d_desc", _lib().qconv_s2d_desc(ctypes.byref(d), ctypes.byref(o)))
    return o


def qconv_quantize_pack_s2d(d: qconv_desc, x, scale: float, out=None, stream=None):
    """fp32/bf16 NHWC x of the original conv -> X2 byte codes [n, h2, w2, c2]."""
    import torch
    assert x.is_cuda and x.is_contiguous() and x.dtype in (torch.float32, torch.bfloat16)
    o = qconv_s2d_desc(d)
    if out is None:
        out = torch.empty((o.n, o.h, o.w, o.c), dtype=torch.uint8, device=x.device)
    _check("qconv_quantize_pack_s2d", _lib().qconv_quantize_pack_s2d(
        ctypes.byref(d), _ptr(x), QC_BF16 if x.dtype == torch.bfloat16 else QC_F32, float(scale),
        _ptr(out), _stream(stream)))
    return out


def qconv_prepare_weights_s2d(d: qconv_desc, w, out=None, stream=None):
    import torch
    nb = int(_lib().qconv_prepared_weight_bytes_s2d(ctypes.byref(d)))
    if nb == 0:
        raise QConvError("qconv_prepare_weights_s2d", 2)
    if out is None:
        out = torch.empty(nb, dtype=torch.uint8, device=w.device)
    _check("qconv_prepare_weights_s2d", _lib().qconv_prepare_weights_s2d(
        ctypes.byref(d), _ptr(w), _ptr(out), _stream(stream)))
    return out


def qconv_debug_im2col_tile(d: qconv_desc, x, m0: int, r: int, s: int, c_byte: int,
                            box_bytes: int, stream=None):
    import torch
    out = torch.empty((128, box_bytes), dtype=torch.uint8, device=x.device)
    _check("qconv_debug_im2col_tile", _lib().qconv_debug_im2col_tile(
        ctypes.byref(d), _ptr(x), int(m0), int(r), int(s), int(c_byte), int(box_bytes),
        _ptr(out), _stream(stream)))
    return out


# --------------------------------------------------------------------------- layer object
@dataclass
class QConv2d:
    """A quantized conv layer resident on one GPU: prepared weights, bias and
    requant parameters live in HBM; __call__ enqueues one qconv2d_forward."""
    desc: qconv_desc
    w_prep: object
    bias: object
    multiplier: object
    shift: object
    workspace: object = None
    scale: object = None          # float outputs: per-channel dequantization scale

    @classmethod
    def create(cls, desc: qconv_desc, w_bytes, bias, multiplier, shift, device="cuda",
               stream=None, scale=None):
        import torch
        w_dev = torch.as_tensor(np.ascontiguousarray(w_bytes)).to(device)
        w_prep = qconv_prepare_weights(desc, w_dev, stream=stream)
        d = qconv_desc.from_buffer_copy(desc)
        d.w_prepared = 1
        b = None if bias is None else torch.as_tensor(np.asarray(bias, np.int32)).to(device)
        m = None if multiplier is None else torch.as_tensor(np.asarray(multiplier, np.int32)).to(device)
        s = None if shift is None else torch.as_tensor(np.asarray(shift, np.int32)).to(device)
        ws = qconv2d_workspace_size(d)
        wsb = torch.empty(ws, dtype=torch.uint8, device=device) if ws else None
        sc = None if scale is None else torch.as_tensor(np.asarray(scale, np.float32)).to(device)
        return cls(d, w_prep, b, m, s, wsb, sc)

    def __call__(self, x, y=None, stream=None):
        if self.desc.y_t in (QC_F32_OUT, QC_BF16_OUT):
            return qconv2d_forward_dequant(self.desc, x, self.w_prep, self.bias, self.scale, y=y,
                                           workspace=self.workspace, stream=stream)
        return qconv2d_forward(self.desc, x, self.w_prep, self.bias, self.multiplier, self.shift,
                               y=y, workspace=self.workspace, stream=stream)


__all__ = ["qconv_quantize_pack", "qconv_requant_params", "qconv_prepare_weights",
           "qconv2d_forward_dequant", "qconv2d_forward_quantize", "qconv_debug_plan", "qconv_debug_plan_quantize", "qconv_plan_candidates",
           "qconv_plan_set", "qconv_plan_clear", "qconv_autotune", "qconv_plan",
           "QC_F32_OUT", "QC_BF16_OUT", "QC_ROUND_SINGLE", "QC_ROUND_TFLITE",
           "QC_KERNEL_AUTO", "QC_KERNEL_IM2COL", "QC_KERNEL_PAIR", "QC_KERNEL_HALO", "QC_KERNEL_HALO_T",
           "QC_KERNEL_CHANNEL",
           "qconv_s2d_desc", "qconv_quantize_pack_s2d", "qconv_prepare_weights_s2d",
           "qconv_prepared_weight_bytes", "qconv2d_workspace_size", "qconv2d_forward",
           "qconv_debug_im2col_tile", "make_desc", "qconv_desc", "QConv2d", "QConvError",
           "QC_U4", "QC_S4", "QC_U8", "QC_S8", "QC_S32", "out_hw", "lib_path"]

_lib()   # fail loudly at import if the CUDA library is missing
