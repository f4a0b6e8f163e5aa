"""Device time of one 3x3/2 max-pool node (NHWC bf16): CUDA graph of 10 launches, L2 flushed before
each replay.    python tools/pool_time.py N H W C"""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_zhanghl21_b200 import duet  # noqa: E402

N, H, W, C = (int(v) for v in sys.argv[1:5])
Ho, Wo = (H - 1) // 2 + 1, (W - 1) // 2 + 1
g = duet.Graph(f"%x = input() : bf16[{N},{H},{W},{C}]\n%y = maxpool(%x) {{k=3, stride=2, pad=1}} : "
               f"bf16[{N},{Ho},{Wo},{C}]\noutput %y\n")
x = torch.randn(N, H, W, C, device="cuda").to(torch.bfloat16)
y = torch.empty(N, Ho, Wo, C, device="cuda", dtype=torch.bfloat16)
flush = torch.empty(128 << 20, dtype=torch.float32, device="cuda")
st = torch.cuda.Stream()
with torch.cuda.stream(st):
    g.node_run("y", [x], y, st)
    st.synchronize()
    gr = torch.cuda.CUDAGraph()
    with torch.cuda.graph(gr, stream=st):
        for _ in range(10):
            g.node_run("y", [x], y, torch.cuda.current_stream())
ts = []
for _ in range(10):
    flush.zero_()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(st):
        e0.record(st)
        gr.replay()
        e1.record(st)
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1) * 1e3 / 10)
us = statistics.median(ts)
byt = (x.numel() + y.numel()) * 2
print(f"maxpool N{N} H{H} W{W} C{C}: {us:.1f} us, {byt / us / 1e3:.0f} GB/s (input + output bytes)")
