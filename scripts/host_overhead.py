"""Host-side cost of one public-API call (python binding -> C ABI -> launch), per layer kind:
wall time of N back-to-back qconv2d_forward calls on small shapes (GPU work ~ few us, so the
loop is host-bound).  python scripts/host_overhead.py"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc  # noqa: E402
import workloads as W  # noqa: E402

for name, shape in [("1x1", (1, 7, 7, 512, 2048, 1, 1, 1, 0)), ("3x3", (1, 7, 7, 512, 512, 3, 3, 1, 1)),
                    ("halo", (1, 56, 56, 64, 64, 3, 3, 1, 1))]:
    n, h, w, c, k, r, s, st, pad = shape
    cs = W.ConvShape(name, n, h, w, c, k, r, s, st, pad)
    li = W.make_layer_inputs(cs, 8, seed=1)
    m, sh = qc.qconv_requant_params(li.s_x, li.s_w, li.s_y)
    d = qc.make_desc(n, h, w, c, k, r, s, stride=st, pad=pad, x_t=li.x_t, w_t=li.w_t, y_t=li.y_t,
                     clamp_lo=li.clamp_lo, clamp_hi=li.clamp_hi)
    x = torch.from_numpy(li.x_bytes).cuda()
    wt = qc.qconv_prepare_weights(d, torch.from_numpy(li.w_bytes).cuda())
    d.w_prepared = 1
    b, mm, nn = (torch.from_numpy(a).cuda() for a in (li.bias, m, sh))
    y = qc.qconv2d_forward(d, x, wt, b, mm, nn)
    lib = qc._lib()
    import ctypes
    args = (ctypes.byref(d), x.data_ptr(), wt.data_ptr(), b.data_ptr(), mm.data_ptr(), nn.data_ptr(),
            y.data_ptr(), None, 0, torch.cuda.current_stream().cuda_stream)
    for _ in range(50):
        lib.qconv2d_forward(*args)
    torch.cuda.synchronize()
    N = 2000
    t0 = time.perf_counter()
    for _ in range(N):
        lib.qconv2d_forward(*args)
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    t3 = time.perf_counter()
    for _ in range(N):
        qc.qconv2d_forward(d, x, wt, b, mm, nn, y=y)
    t4 = time.perf_counter()
    torch.cuda.synchronize()
    print(f"{name}: C ABI call {1e6 * (t1 - t0) / N:.1f} us/call (drain {1e3 * (t2 - t1):.1f} ms); "
          f"python binding {1e6 * (t4 - t3) / N:.1f} us/call; plan {qc.qconv_debug_plan(d)['kernel_name']}")
