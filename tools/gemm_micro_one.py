"""A few launches of one GEMM node (or the c2 deep gather, or an fp32 conv) for ncu captures.
  python tools/gemm_micro_one.py M N K [f32] | gather | conv N H W C Co k stride pad [f32]"""
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
elif sys.argv[1] == "conv":
    N, H, Wd, C, Co, k, s, p = (int(v) for v in sys.argv[2:10])
    dt = sys.argv[10] if len(sys.argv) > 10 else "bf16"
    tdt = torch.float32 if dt == "f32" else torch.bfloat16
    Ho, Wo = (H + 2 * p - k) // s + 1, (Wd + 2 * p - k) // s + 1
    ir = (f"param @W : {dt}[{Co},{k},{k},{C}]\nparam @g : f32[{Co}]\nparam @b : f32[{Co}]\nparam @m : f32[{Co}]\n"
          f"param @v : f32[{Co}]\n%x = input() : {dt}[{N},{H},{Wd},{C}]\n"
          f"%y = conv2d_bn(%x, @W, @g, @b, @m, @v) {{stride={s}, pad={p}, act=relu}} : {dt}[{N},{Ho},{Wo},{Co}]\n"
          f"output %y\n")
    g = duet.Graph(ir)
    g.bind_all({"W": (torch.randn(Co, k, k, C, device="cuda") * 0.05).to(tdt), "g": torch.ones(Co, device="cuda"),
                "b": torch.zeros(Co, device="cuda"), "m": torch.zeros(Co, device="cuda"),
                "v": torch.ones(Co, device="cuda")})
    x = torch.randn(N, H, Wd, C, device="cuda").to(tdt)
    y = torch.empty(N, Ho, Wo, Co, device="cuda", dtype=tdt)
    for _ in range(4):
        g.node_run("y", [x], y)
else:
    M, N, K = (int(v) for v in sys.argv[1:4])
    dt = sys.argv[4] if len(sys.argv) > 4 else "bf16"
    tdt = torch.float32 if dt == "f32" else torch.bfloat16
    ir = (f"param @W : {dt}[{N},{K}]\nparam @b : f32[{N}]\n%x = input() : {dt}[{M},{K}]\n"
          f"%y = linear(%x, @W, @b) {{act=relu}} : {dt}[{M},{N}]\noutput %y\n")
    g = duet.Graph(ir)
    g.bind_all({"W": (torch.randn(N, K, device="cuda") * 0.05).to(tdt), "b": torch.zeros(N, device="cuda")})
    x = torch.randn(M, K, device="cuda").to(tdt)
    y = torch.empty(M, N, device="cuda", dtype=tdt)
    for _ in range(4):
        g.node_run("y", [x], y)
torch.cuda.synchronize()
