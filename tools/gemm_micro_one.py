"""A few launches of one GEMM node (or the c2 deep gather) for ncu captures.
  python tools/gemm_micro_one.py M N K | gather"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_zhanghl21_b200 import duet  # noqa: E402
from paper_conf_ipps_zhanghl21_b200 import workloads as W  # noqa: E402
from paper_conf_ipps_zhanghl21_b200.harness import materialize  # noqa: E402

if sys.argv[1] == "gather":
    wl = W.build("c2")
    g = duet.Graph(wl.ir)
    g.bind_all(materialize(wl.params, "cuda"))
    raw = wl.inputs["raw"].materialize("cuda")
    ids = torch.empty(raw.shape, dtype=torch.int32, device="cuda")
    g.node_run("ids", [raw], ids)
    X = torch.empty((raw.shape[0], raw.shape[1] * 64), dtype=torch.bfloat16, device="cuda")
    for _ in range(4):
        g.node_run("deep_x", [ids], X)
else:
    M, N, K = (int(v) for v in sys.argv[1:4])
    ir = (f"param @W : bf16[{N},{K}]\nparam @b : f32[{N}]\n%x = input() : bf16[{M},{K}]\n"
          f"%y = linear(%x, @W, @b) {{act=relu}} : bf16[{M},{N}]\noutput %y\n")
    g = duet.Graph(ir)
    g.bind_all({"W": (torch.randn(N, K, device="cuda") * 0.05).to(torch.bfloat16), "b": torch.zeros(N, device="cuda")})
    x = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    y = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    for _ in range(4):
        g.node_run("y", [x], y)
torch.cuda.synchronize()
