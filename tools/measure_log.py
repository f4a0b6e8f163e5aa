"""Log measured-mode Step 3 costs for one config (DUET_MEASURE_LOG=1 python tools/measure_log.py c5)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

from paper_conf_ipps_zhanghl21_b200 import duet
from paper_conf_ipps_zhanghl21_b200 import workloads as W
from paper_conf_ipps_zhanghl21_b200.harness import Session

wl = W.build(sys.argv[1])
sess = Session(wl, n_slots=2, profile=dict(warmup=2, samples=10, reps=3))
torch.cuda.synchronize()
t = time.time()
s = sess.schedule(duet.GREEDY_CORRECTION, measured=True, samples=int(os.environ.get("SAMPLES", "10")), warmup=1)
print("measured schedule", s.export(), s.measured_ns, s.evaluations, f"{time.time() - t:.1f}s", flush=True)
