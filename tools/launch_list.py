"""The kernels of K DUET steps of a config, for the ncu launch list (profiles/<tag>_launches.md):

    ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv \
        --log-file gpurun_out/launches.csv python tools/launch_list.py c5 3

Builds the session as bench.py does (model-mode greedy-correction schedule, fast profile), then
wraps K steps in cudaProfilerStart/Stop so ncu records exactly those launches.  ncu serialises
and cold-starts every kernel, so per-launch times are not the step's; the shares are what
bench.py's roofline is checked against."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_ipps_zhanghl21_b200 import workloads as W  # noqa: E402
from paper_conf_ipps_zhanghl21_b200.harness import Session, materialize  # noqa: E402


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "c5"
    k = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    wl = W.build(cfg)
    sess = Session(wl, n_slots=2, profile=dict(warmup=2, samples=5, reps=2))
    s = sess.schedule()
    inputs = list(materialize(wl.inputs, "cuda").values())
    outs = sess.outputs()
    for _ in range(2):
        sess.run(s, inputs, outs)
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    for _ in range(k):
        sess.run(s, inputs, outs)
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    print("schedule", s.export(), "launches per step", s.launch_count())


if __name__ == "__main__":
    main()
