"""Time one fp32 linear node (3xTF32, gemm_tf32.cu) under DUET_GEMM_DBG settings, each in a fresh
process; prints us per launch (CUDA graph of back-to-back launches) and the error vs float64.
  python tools/tf32_time.py M N K bn dbg..."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
from paper_conf_ipps_zhanghl21_b200 import duet
from tests.helpers import rel_err
M, N, K = map(int, sys.argv[2:5])
ir = (f"param @W : f32[{N},{K}]\nparam @b : f32[{N}]\n%x = input() : f32[{M},{K}]\n"
      f"%y = linear(%x, @W, @b) {{act=relu}} : f32[{M},{N}]\noutput %y\n")
g_ = torch.Generator().manual_seed(1)
x = ((torch.rand(M, K, generator=g_, dtype=torch.float64) * 2 - 1)).float()
W = ((torch.rand(N, K, generator=g_, dtype=torch.float64) * 2 - 1) / K ** 0.5).float()
b = ((torch.rand(N, generator=g_, dtype=torch.float64) * 2 - 1) * 0.1).float()
g = duet.Graph(ir)
g.bind_all({"W": W.cuda(), "b": b.cuda()})
xd = x.cuda()
y = torch.empty(M, N, device="cuda")
st = torch.cuda.Stream()
with torch.cuda.stream(st):
    for _ in range(3):
        g.node_run("y", [xd], y, st)
    st.synchronize()
    gr = torch.cuda.CUDAGraph()
    with torch.cuda.graph(gr, stream=st):
        for _ in range(20):
            g.node_run("y", [xd], y, torch.cuda.current_stream())
    ts = []
    for _ in range(10):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st); gr.replay(); e1.record(st); st.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3 / 20)
g.node_run("y", [xd], y, st)
st.synchronize()
want = torch.relu(x.double() @ W.double().T + b.double()).numpy()
us = sorted(ts)[len(ts) // 2]
print(f"{us:.2f} us  {2 * M * N * K / us / 1e6:.1f} TFLOP/s  rel err {rel_err(y.cpu().numpy(), want):.3e}")
'''
M, N, K, bn = sys.argv[1:5]
for dbg in sys.argv[5:]:
    env = dict(os.environ, DUET_GEMM_DBG=dbg, DUET_GEMM_BN=bn)
    r = subprocess.run([sys.executable, "-c", CHILD, ROOT, M, N, K], env=env, capture_output=True, text=True)
    print(f"M{M} N{N} K{K} bn{bn} dbg {dbg}: {r.stdout.strip()} {r.stderr.strip()[-300:]}", flush=True)
