import sys, torch
sys.path.insert(0, 'tools')
from gemm_micro import warm, sm_clock
warm(1.0)
print("clk", sm_clock())
for (M, N, K) in [(2048, 1024, 1664), (2048, 512, 1024), (2048, 256, 512), (4096, 1024, 1664), (16384, 2048, 256),
                  (256, 2048, 512), (4096, 4096, 4096), (8192, 8192, 8192)]:
    a = torch.randn(M, K, device="cuda", dtype=torch.bfloat16)
    w = torch.randn(N, K, device="cuda", dtype=torch.bfloat16)
    for _ in range(20): a @ w.T
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    with torch.cuda.graph(g, stream=s):
        for _ in range(20): y = a @ w.T
    for _ in range(5): g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record(); [g.replay() for _ in range(10)]; e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 200
    print(f"cuBLAS M={M} N={N} K={K} {ms*1e3:8.2f} us {2*M*N*K/ms/1e9:8.1f} TF/s")
