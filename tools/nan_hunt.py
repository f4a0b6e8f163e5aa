"""After a c3 session, run c4 with every ResNet add/pool/stem node exposed as an output and report
the first node whose output contains NaN/Inf."""
import sys, os, gc, re
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_zhanghl21_b200 import workloads as W
from paper_conf_ipps_zhanghl21_b200.workloads import Workload
from paper_conf_ipps_zhanghl21_b200.harness import Session, materialize
for pre in sys.argv[1:]:
    wl = W.build(pre, branch_outputs=True)
    sess = Session(wl, n_slots=2, profile=dict(warmup=1, samples=2, reps=2))
    inputs = list(materialize(wl.inputs, "cuda").values())
    outs = sess.outputs()
    sess.run(sess.schedule(), inputs, outs)
    torch.cuda.synchronize()
    del sess, inputs, outs
    gc.collect()
wl = W.build("c4", branch_outputs=True)
names = [m.group(1) for m in re.finditer(r"^%(cnn_\w+) = (conv2d_bn|maxpool|add|avgpool)", wl.ir, re.M)
         if m.group(2) != "conv2d_bn" or m.group(1).endswith("stem")]
decl = {m.group(1): (m.group(2), tuple(int(x) for x in m.group(3).split(",")))
        for m in re.finditer(r"^%(\w+) = .*: (\w+)\[([0-9,]*)\]$", wl.ir, re.M)}
lines = wl.ir.splitlines()
oi = next(i for i, l in enumerate(lines) if l.startswith("output "))
lines[oi] += "".join(f", %{n}" for n in names if n not in lines[oi])
order = {m.group(1): i for i, m in enumerate(re.finditer(r"^%(\w+) =", wl.ir, re.M))}
outs_spec = sorted(set([o[0] for o in wl.outputs] + names), key=lambda n: order[n])
wl2 = Workload(wl.name, "\n".join(lines) + "\n", wl.params, wl.inputs,
               [(n, decl[n][0], decl[n][1]) for n in outs_spec], wl.batch, {})
sess = Session(wl2, n_slots=int(os.environ.get("SLOTS", "2")), profile=dict(warmup=1, samples=2, reps=2))
inputs = list(materialize(wl2.inputs, "cuda").values())
outs = sess.outputs()
sess.run(sess.schedule(), inputs, outs)
torch.cuda.synchronize()
for (n, _, _), o in zip(wl2.outputs, outs):
    bad = (~torch.isfinite(o.float())).sum().item()
    print(f"{n:20s} nonfinite={bad:8d} max={o.float().abs().nan_to_num(0).max().item():.3f}")
