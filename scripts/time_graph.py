"""Time the bench trunk step as one CUDA graph with no events inside (debug: PDL on/off)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
bits = int(sys.argv[1]) if len(sys.argv) > 1 else 4
tr = bench.Trunk(bits, 256, "cuda")
s = torch.cuda.Stream()
with torch.cuda.stream(s):
    for _ in range(3): tr.step()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        tr.step()
    for _ in range(5): g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(30): g.replay()
    e1.record()
torch.cuda.synchronize()
print(f"{bits}-bit graph step {e0.elapsed_time(e1) / 30:.4f} ms  PDL={'off' if os.environ.get('QC_NO_PDL') else 'on'}")
