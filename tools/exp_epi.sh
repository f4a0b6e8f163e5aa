mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "gather_fused" > gpurun_out/gf2_tests.log 2>&1; echo rc=$? >> gpurun_out/gf2_tests.log
python tools/gemm_trace.py 2048 1024 1664 > gpurun_out/trace_epi.log 2>&1
DUET_TMA_STORE=0 python tools/gemm_trace.py 2048 1024 1664 > gpurun_out/trace_epi_notma.log 2>&1
python tools/gemm_trace.py 2048 256 512 > gpurun_out/trace_epi_fc3.log 2>&1
python - <<'PY' > gpurun_out/gf_micro.log 2>&1
import sys, torch
sys.path.insert(0, "."); sys.path.insert(0, "tools")
from gemm_micro import warm
from paper_conf_ipps_zhanghl21_b200 import duet
warm(1.0)
B, F, R, N = 2048, 26, 1000000, 1024
ir = (f"param @E : bf16[{F},{R},64]\nparam @W : bf16[{N},{64 * F}]\nparam @b : f32[{N}]\n"
      f"%ids = input() : i32[{B},{F}]\n%x = gather_concat(%ids, @E) : bf16[{B},{64 * F}]\n"
      f"%y = linear(%x, @W, @b) {{act=relu}} : bf16[{B},{N}]\noutput %y\n")
g = duet.Graph(ir)
g.bind_all({"E": torch.randn(F, R, 64, device="cuda").to(torch.bfloat16), "W": (torch.randn(N, 64*F, device="cuda")*0.02).to(torch.bfloat16), "b": torch.zeros(N, device="cuda")})
s = g.partition().profile_from_table([0], [[1000]]).schedule()
st = torch.cuda.Stream()
ids = torch.randint(0, R, (B, F), device="cuda", dtype=torch.int32)
y = torch.empty(B, N, device="cuda", dtype=torch.bfloat16)
x = torch.empty(B, 64*F, device="cuda", dtype=torch.bfloat16)
def t(fn, reps=50):
    for _ in range(5): fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    with torch.cuda.stream(st):
        e0.record(st)
        for _ in range(reps): fn()
        e1.record(st)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3
print("fused gather+fc1 (graph launch each)", t(lambda: s.run([(0, st)], [ids], [y])), "us")
print("gather node", t(lambda: g.node_run("x", [ids], x, st)), "us")
print("fc1 node", t(lambda: g.node_run("y", [x], y, st)), "us")
PY
