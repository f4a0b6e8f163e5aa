"""c1 placement experiment: every assignment of c1's 4 subgraphs to 2 slots, measured warm (as in
tools/fig13.py), with the session's slot priorities (home normal, other high), equal priorities,
and swapped priorities."""
import itertools, json, os, statistics, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
from paper_conf_ipps_zhanghl21_b200 import duet
from paper_conf_ipps_zhanghl21_b200 import workloads as W
from paper_conf_ipps_zhanghl21_b200.harness import Session, materialize

cfg = sys.argv[1] if len(sys.argv) > 1 else "c1"
wl = W.build(cfg)
sess = Session(wl, n_slots=2, profile=dict(warmup=5, samples=50, reps=10, calibrate_comm=True))
inputs = list(materialize(wl.inputs, "cuda").values())
outs = sess.outputs()
torch.cuda.synchronize()
variants = {"session (0,-1)": sess.slots,
            "equal (0,0)": [(0, torch.cuda.Stream(priority=0)), (0, torch.cuda.Stream(priority=0))],
            "swapped (-1,0)": [(0, torch.cuda.Stream(priority=-1)), (0, torch.cuda.Stream(priority=0))]}
n = sess.part.n_sg
res = {}
for vname, slots in variants.items():
    home = slots[0][1]
    home.wait_stream(torch.cuda.current_stream())
    for a in itertools.product(range(2), repeat=n):
        s = sess.prof.schedule(mode=duet.FIXED, fixed=list(a))
        for _ in range(10):
            s.run(slots, inputs, outs)
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(201)]
        ev[0].record(home)
        for k in range(200):
            s.run(slots, inputs, outs)
            ev[k + 1].record(home)
        home.synchronize()
        ms = statistics.median(ev[k].elapsed_time(ev[k + 1]) for k in range(200))
        res.setdefault(str(list(a)), {})[vname] = round(ms * 1e3, 2)
        torch.cuda.synchronize()
for a, r in res.items():
    print(a, json.dumps(r))
gc = sess.schedule(duet.GREEDY_CORRECTION, measured=True, samples=20)
print("measured greedy-correction:", gc.export()["slot_of"], gc.measured_ns)
