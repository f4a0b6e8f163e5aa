# measured Step 3 with cold replays (DUET_MEASURE_FLUSH=1, default) vs back-to-back warm ones (0)
for c in c5 c4 c2; do
  for m in 1 0 1 0; do
    echo -n "$c flush=$m: "
    DUET_MEASURE_FLUSH=$m timeout 500 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline --per-config none \
      --tail-samples 200 | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print({k: d.get(k) for k in ('p50_ms','serial_p50_ms','speedup_vs_serial')}, d['schedule']['slot_of'], d['schedule']['measured_ns'])"
  done
done
