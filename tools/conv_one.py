"""One conv2d_bn node at a given shape, for ncu / timing (bf16, NHWC, BN folded, ReLU).

    python tools/conv_one.py N H C Co k stride pad [reps] [residual]
With CONV_ONE_GRAPH=1: a CUDA graph of 10 back-to-back launches per replay (no host latency in
the figure; only the first launch of a replay starts cold).
"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_ipps_zhanghl21_b200 import duet  # noqa: E402


def main():
    N, H, C, Co, k, s, p = (int(v) for v in sys.argv[1:8])
    reps = int(sys.argv[8]) if len(sys.argv) > 8 else 20
    Ho = (H + 2 * p - k) // s + 1
    ir = (f"param @W : bf16[{Co},{k},{k},{C}]\nparam @g : f32[{Co}]\nparam @b : f32[{Co}]\nparam @m : f32[{Co}]\n"
          f"param @v : f32[{Co}]\n%x = input() : bf16[{N},{H},{H},{C}]\n"
          f"%y = conv2d_bn(%x, @W, @g, @b, @m, @v) {{stride={s}, pad={p}, act=relu}} : bf16[{N},{Ho},{Ho},{Co}]\n"
          "output %y\n")
    g = duet.Graph(ir)
    gen = torch.Generator().manual_seed(0)
    g.bind_all({"W": (torch.randn(Co, k, k, C, generator=gen) * (2 / (k * k * C)) ** 0.5).to(torch.bfloat16).cuda(),
                "g": torch.ones(Co).cuda(), "b": torch.zeros(Co).cuda(), "m": torch.zeros(Co).cuda(),
                "v": torch.ones(Co).cuda()})
    x = torch.randn(N, H, H, C, generator=gen).to(torch.bfloat16).cuda()
    y = torch.empty(N, Ho, Ho, Co, dtype=torch.bfloat16, device="cuda")
    flush = torch.empty(128 << 20, dtype=torch.float32, device="cuda")
    st = torch.cuda.Stream()
    ts = []
    if os.environ.get("CONV_ONE_GRAPH") == "1":
        with torch.cuda.stream(st):
            g.node_run("y", [x], y, st)
            st.synchronize()
            gr = torch.cuda.CUDAGraph()
            with torch.cuda.graph(gr, stream=st):
                for _ in range(10):
                    g.node_run("y", [x], y, torch.cuda.current_stream())
        for i in range(reps):
            flush.zero_()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            with torch.cuda.stream(st):
                e0.record(st)
                gr.replay()
                e1.record(st)
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e3 / 10)
        reps = -2
    for i in range(reps + 2):
        flush.zero_()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        g.node_run("y", [x], y, st)
        e1.record(st)
        torch.cuda.synchronize()
        if i >= 2:
            ts.append(e0.elapsed_time(e1) * 1e3)
    fl = 2 * N * Ho * Ho * Co * C * k * k
    us = statistics.median(ts)
    print(f"conv N{N} H{H} C{C} Co{Co} k{k} s{s} p{p}: {us:.2f} us  {fl / us / 1e6:.1f} TFLOP/s")


if __name__ == "__main__":
    main()
