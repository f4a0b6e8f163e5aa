import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_zhanghl21_b200 import workloads as W
from paper_conf_ipps_zhanghl21_b200.harness import Session, materialize
cfg = sys.argv[1] if len(sys.argv) > 1 else "c4"
wl = W.build(cfg, branch_outputs=True)
sess = Session(wl, n_slots=2,
               profile=dict(warmup=1, samples=1, reps=1))
inputs = list(materialize(wl.inputs, "cuda").values())
outs = sess.outputs()
sess.run(sess.schedule(), inputs, outs)
torch.cuda.synchronize()
print("ok", [float(o.float().abs().max()) for o in outs])
