# DUET over 2 / 3 / 4 CUDA-stream slots (bench.py --slots), configs c2-c5
for c in c5 c4 c2 c3; do
  for n in 2 3 4; do
    echo "== $c slots=$n"
    timeout 400 python bench.py --config $c --slots $n --steps 100 --warmup 10 --no-cpu-baseline --per-config none \
      --tail-samples 200 | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print({k: d.get(k) for k in ('p50_ms','serial_p50_ms','speedup_vs_serial')}, d['schedule']['slot_of'])"
  done
done
