import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_hanhyylhgwwlq20_b200 as qc
d = qc.make_desc(256, 224, 224, 3, 64, 7, 7, stride=2, pad=3, x_t=qc.QC_U4, w_t=qc.QC_S8, y_t=qc.QC_U4)
x = torch.relu(torch.randn(256, 224, 224, 3, device="cuda"))
y = qc.qconv_quantize_pack_s2d(d, x, 0.2)
for _ in range(3): qc.qconv_quantize_pack_s2d(d, x, 0.2, out=y)
e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(20): qc.qconv_quantize_pack_s2d(d, x, 0.2, out=y)
e1.record(); torch.cuda.synchronize()
us = e0.elapsed_time(e1) / 20 * 1e3
print(f"quantize_s2d {us:.1f} us  {(x.numel()*4 + y.numel())/us/1e3:.0f} GB/s")
