"""A few launches of one recurrent node (no timestamps) for ncu captures.
  python tools/rnn_trace_plain.py lstm|gru B H E S"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_zhanghl21_b200 import duet  # noqa: E402

kind = sys.argv[1]
B, H, E, S = (int(x) for x in sys.argv[2:6])
G = 4 if kind == "lstm" else 3
ir = (f"param @Wih : bf16[{G * H},{E}]\nparam @Whh : bf16[{G * H},{H}]\nparam @bih : f32[{G * H}]\n"
      f"param @bhh : f32[{G * H}]\n%x = input() : bf16[{S},{B},{E}]\n"
      f"%y = {kind}(%x, @Wih, @Whh, @bih, @bhh) : bf16[{B},{H}]\noutput %y\n")
g = duet.Graph(ir)
k = 1.0 / H ** 0.5
g.bind_all({"Wih": ((torch.rand(G * H, E, device="cuda") * 2 - 1) * k).to(torch.bfloat16),
            "Whh": ((torch.rand(G * H, H, device="cuda") * 2 - 1) * k).to(torch.bfloat16),
            "bih": torch.zeros(G * H, device="cuda"), "bhh": torch.zeros(G * H, device="cuda")})
x = torch.randn(S, B, E, device="cuda").to(torch.bfloat16)
y = torch.empty(B, H, device="cuda", dtype=torch.bfloat16)
for _ in range(3):
    g.node_run("y", [x], y)
torch.cuda.synchronize()
