"""Device time of one recurrent node launch (CUDA events around node_run; warm).
  python tools/rnn_time.py lstm|gru B H E S"""
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
st = torch.cuda.Stream()
for _ in range(3):
    g.node_run("y", [x], y, st)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
with torch.cuda.stream(st):
    e0.record(st)
    for _ in range(5):
        g.node_run("y", [x], y, st)
    e1.record(st)
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 5
fl = 2 * B * G * H * (E + H) * S
print(f"{kind} B{B} H{H} E{E} S{S} env BN={os.environ.get('DUET_RNN_BN', '-')} GRID={os.environ.get('DUET_RNN_GRID', '-')}: "
      f"{ms * 1e3:.1f} us, {ms * 1e3 / S:.2f} us/step, {fl / ms / 1e9:.0f} TFLOP/s")
