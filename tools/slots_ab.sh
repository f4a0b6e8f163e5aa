# c5 on 2 vs 3 CUDA-stream slots, alternating, same box
for r in 1 2 3; do
  for n in 2 3; do
    echo -n "c5 slots=$n: "
    timeout 400 python bench.py --config c5 --slots $n --steps 100 --warmup 10 --no-cpu-baseline --per-config none \
      --tail-samples 200 | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print({k: d.get(k) for k in ('p50_ms','serial_p50_ms','speedup_vs_serial')}, d['schedule']['slot_of'])"
  done
done
