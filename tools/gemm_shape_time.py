"""Device time of one linear node (bf16, ReLU) at a given shape: CUDA graph of 10 launches, L2 flushed
before each replay.  Kernel choice through the usual env switches (DUET_GEMM=1: one-CTA tiles,
DUET_GEMM_BN: tile width).    python tools/gemm_shape_time.py M N K [reps]"""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_zhanghl21_b200 import duet  # noqa: E402

M, N, K = (int(v) for v in sys.argv[1:4])
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 10
ir = (f"param @W : bf16[{N},{K}]\nparam @b : f32[{N}]\n%x = input() : bf16[{M},{K}]\n"
      f"%y = linear(%x, @W, @b) {{act=relu}} : bf16[{M},{N}]\noutput %y\n")
g = duet.Graph(ir)
g.bind_all({"W": (torch.randn(N, K, device="cuda") * 0.05).to(torch.bfloat16), "b": torch.zeros(N, device="cuda")})
x = torch.randn(M, K, device="cuda").to(torch.bfloat16)
y = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
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
for _ in range(reps):
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
print(f"gemm M{M} N{N} K{K} GEMM={os.environ.get('DUET_GEMM', '-')} BN={os.environ.get('DUET_GEMM_BN', '-')}: "
      f"{us:.1f} us, {2 * M * N * K / us / 1e6:.0f} TFLOP/s")
