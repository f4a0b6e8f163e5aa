import sys, os, gc
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_zhanghl21_b200 import duet, workloads as W
from paper_conf_ipps_zhanghl21_b200.harness import Session, materialize
if len(sys.argv) > 1 and sys.argv[1] == "dirty":
    wl = W.build("c3")
    s = Session(wl, n_slots=2, profile=dict(warmup=1, samples=2, reps=2))
    ins = list(materialize(wl.inputs, "cuda").values()); outs = s.outputs()
    s.run(s.schedule(), ins, outs); torch.cuda.synchronize(); del s, ins, outs; gc.collect()
N, H, C, Co = 64, 224, 3, 64
ir = ("param @W : bf16[64,7,7,3]\nparam @g : f32[64]\nparam @b : f32[64]\nparam @m : f32[64]\nparam @v : f32[64]\n"
      "%x = input() : bf16[64,224,224,3]\n%y = conv2d_bn(%x, @W, @g, @b, @m, @v) {stride=2, pad=3, act=relu} : bf16[64,112,112,64]\noutput %y\n")
g = duet.Graph(ir)
Wt = (torch.randn(64, 7, 7, 3, device="cuda") * 0.1).bfloat16()
ones = torch.ones(64, device="cuda"); zeros = torch.zeros(64, device="cuda")
g.bind_all({"W": Wt, "g": ones, "b": zeros, "m": zeros, "v": ones})
x = torch.randn(64, 224, 224, 3, device="cuda").bfloat16()
for rep in range(3):
    y = torch.empty(64, 112, 112, 64, device="cuda", dtype=torch.bfloat16)
    g.node_run("y", [x], y); torch.cuda.synchronize()
    ref = torch.relu(torch.nn.functional.conv2d(x.float().permute(0, 3, 1, 2), Wt.float().permute(0, 3, 1, 2), stride=2, padding=3)).permute(0, 2, 3, 1) / (1 + 1e-5) ** 0.5
    bad = (~torch.isfinite(y.float())).sum().item()
    err = ((y.float() - ref).abs().max() / ref.abs().max()).item()
    print(f"rep {rep} nonfinite={bad} err={err:.3e}", flush=True)
