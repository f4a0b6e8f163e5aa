#!/bin/bash
# fp32 mode p50 per config (bench.py --dtype f32), optionally with DUET_TF32=$TF.  Output: gpurun_out/f32_bench.log
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
: > gpurun_out/f32_bench.log
for cfg in ${CFGS:-c1 c2 c3 c4 c5 c6}; do
  line=$(timeout 900 python bench.py --config $cfg --dtype f32 --per-config none --no-cpu-baseline \
         --steps 30 --warmup 3 --tail-samples 0 --profile-samples 20 2>/dev/null | grep '^{' | tail -1)
  echo "$line" >> gpurun_out/f32_bench.jsonl
  python - "$cfg" "$line" >> gpurun_out/f32_bench.log <<'PY'
import json, sys
cfg, line = sys.argv[1:3]
try:
    d = json.loads(line)
    print(f"{cfg} f32: p50 {d['p50_ms']} ms serial {d['serial_p50_ms']} ms launches {d['gpu_launches_per_step']}")
except Exception as e:
    print(f"{cfg} f32: failed {e} {line[:200]}")
PY
done
cat gpurun_out/f32_bench.log
