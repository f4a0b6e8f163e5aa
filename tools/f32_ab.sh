#!/bin/bash
# fp32 mode: 3xTF32 tensor-core contractions (default) vs the CUDA-core kernels (DUET_TF32=0), same
# box, bench.py p50 per config.  Output: gpurun_out/f32_ab.log
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
: > gpurun_out/f32_ab.log
for cfg in c1 c2 c3 c4 c5 c6; do
  for tf in 1 0; do
    line=$(DUET_TF32=$tf timeout 900 python bench.py --config $cfg --dtype f32 --per-config none --no-cpu-baseline \
           --steps 30 --warmup 3 --tail-samples 0 --profile-samples 20 2>/dev/null | grep '^{' | tail -1)
    python - "$cfg" "$tf" "$line" >> gpurun_out/f32_ab.log <<'PY'
import json, sys
cfg, tf, line = sys.argv[1:4]
try:
    d = json.loads(line)
    print(f"{cfg} f32 DUET_TF32={tf}: p50 {d['p50_ms']} ms serial {d['serial_p50_ms']} ms launches {d['gpu_launches_per_step']}")
except Exception as e:
    print(f"{cfg} f32 DUET_TF32={tf}: failed {e} {line[:200]}")
PY
  done
done
cat gpurun_out/f32_ab.log
