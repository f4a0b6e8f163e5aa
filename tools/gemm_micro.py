"""Micro-benchmark of the tcgen05 GEMM tile through duet_node_run (CUDA-graph timed, no host
overhead).  Usage (GPU box): python tools/gemm_micro.py"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_zhanghl21_b200 import duet  # noqa: E402


def time_linear(M, N, K, reps=20, out="bf16"):
    ir = (f"param @W : bf16[{N},{K}]\nparam @b : f32[{N}]\n%x = input() : bf16[{M},{K}]\n"
          f"%y = linear(%x, @W, @b) {{act=relu}} : {out}[{M},{N}]\noutput %y\n")
    g = duet.Graph(ir)
    W = (torch.randn(N, K, device="cuda") * 0.05).to(torch.bfloat16)
    b = torch.zeros(N, device="cuda")
    g.bind_all({"W": W, "b": b})
    x = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    y = torch.empty(M, N, device="cuda", dtype=torch.bfloat16 if out == "bf16" else torch.float32)
    s = torch.cuda.Stream()
    g.node_run("y", [x], y, s)
    torch.cuda.synchronize()
    cg = torch.cuda.CUDAGraph()
    with torch.cuda.graph(cg, stream=s):
        for _ in range(reps):
            g.node_run("y", [x], y, s)
    for _ in range(30):
        cg.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(10):
        cg.replay()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / (10 * reps)
    ref = torch.relu(x.float() @ W.float().T)
    err = (y.float() - ref).abs().max().item() / ref.abs().max().item()
    return ms, 2 * M * N * K / (ms * 1e-3) / 1e12, err


def warm(seconds=1.5):
    import time
    a = torch.randn(8192, 8192, device="cuda", dtype=torch.bfloat16)
    t0 = time.time()
    while time.time() - t0 < seconds:
        for _ in range(10):
            a @ a
        torch.cuda.synchronize()


def sm_clock():
    try:
        import pynvml
        pynvml.nvmlInit()
        return pynvml.nvmlDeviceGetClockInfo(pynvml.nvmlDeviceGetHandleByIndex(0), pynvml.NVML_CLOCK_SM)
    except Exception:
        return -1


if __name__ == "__main__":
    warm()
    print("sm clock after warm-up", sm_clock())
    rows = []
    for (M, N, K) in [(128, 64, 64), (128, 64, 640), (128, 64, 6400), (128, 128, 6400), (128, 256, 6400),
                      (2048, 1024, 1664), (2048, 512, 1024), (2048, 256, 512), (4096, 4096, 4096),
                      (8192, 8192, 8192), (16384, 2048, 256), (256, 2048, 512)]:
        ms, tf, err = time_linear(M, N, K)
        line = f"M={M:6d} N={N:5d} K={K:5d}  {ms * 1e3:9.2f} us  {tf:8.1f} TFLOP/s  err {err:.1e}"
        print(line, flush=True)
