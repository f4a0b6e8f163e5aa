"""Device time of one embed_seq node (token embedding, time-major [S, B, E] out) or the c2-style
gather_concat: CUDA graph of 10 launches, L2 flushed before each replay.
    python tools/embed_time.py S B E [V]"""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_zhanghl21_b200 import duet  # noqa: E402

S, B, E = (int(v) for v in sys.argv[1:4])
V = int(sys.argv[4]) if len(sys.argv) > 4 else 32768
ir = (f"param @E : bf16[{V},{E}]\n%tok = input() : i32[{B},{S}]\n"
      f"%x = embed_seq(%tok, @E) : bf16[{S},{B},{E}]\noutput %x\n")
g = duet.Graph(ir)
g.bind_all({"E": torch.randn(V, E, device="cuda").to(torch.bfloat16)})
tok = torch.randint(0, V, (B, S), device="cuda", dtype=torch.int32)
x = torch.empty(S, B, E, device="cuda", dtype=torch.bfloat16)
flush = torch.empty(128 << 20, dtype=torch.float32, device="cuda")
st = torch.cuda.Stream()
with torch.cuda.stream(st):
    g.node_run("x", [tok], x, st)
    st.synchronize()
    gr = torch.cuda.CUDAGraph()
    with torch.cuda.graph(gr, stream=st):
        for _ in range(10):
            g.node_run("x", [tok], x, torch.cuda.current_stream())
ts = []
for _ in range(10):
    flush.zero_()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(st):
        e0.record(st)
        gr.replay()
        e1.record(st)
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1) * 1e3 / 10)
us = statistics.median(ts)
byt = S * B * E * 2 * 2 + S * B * 4
print(f"embed S{S} B{B} E{E} UNR={os.environ.get('DUET_GATHER_UNR', '4')}: {us:.1f} us, {byt / us / 1e3:.0f} GB/s "
      f"(write + row reads + ids)")
