mkdir -p gpurun_out
python - <<'PY' > gpurun_out/att_prep.log 2>&1
PY
timeout 600 ncu --set full --clock-control none --import-source on -k regex:attention_kernel -s 2 -c 1 -o gpurun_out/att python - <<'PY' > gpurun_out/ncu_att.log 2>&1
import sys, torch
sys.path.insert(0, ".")
from paper_conf_ipps_zhanghl21_b200 import duet
B, S, heads, dh = 1, 128, 12, 64
H = heads * dh
ir = f"%x = input() : bf16[{B*S},{3*H}]\n%y = attention(%x) {{heads={heads}, seq={S}}} : bf16[{B*S},{H}]\noutput %y\n"
g = duet.Graph(ir)
x = torch.randn(B * S, 3 * H, device="cuda").to(torch.bfloat16)
y = torch.empty(B * S, H, device="cuda", dtype=torch.bfloat16)
for _ in range(4):
    g.node_run("y", [x], y)
torch.cuda.synchronize()
PY
ncu -i gpurun_out/att.ncu-rep --page raw --csv > gpurun_out/att_raw.csv 2>/dev/null
ncu -i gpurun_out/att.ncu-rep --page source --csv --print-source sass > gpurun_out/att_sass.csv 2>/dev/null
ncu -i gpurun_out/att.ncu-rep --page details > gpurun_out/att_details.txt 2>/dev/null
