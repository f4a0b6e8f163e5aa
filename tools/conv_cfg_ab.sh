# whole-config A/B of the conv CTAs-per-SM defaults (DUET_CONV_OCC128: 0 auto, 1 one CTA)
for c in c4 c5; do
  for mode in 0 1 0 1; do
    echo -n "$c occ128=$mode: "
    DUET_CONV_OCC128=$mode timeout 400 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline --per-config none \
      --tail-samples 200 | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print({k: d.get(k) for k in ('p50_ms','serial_p50_ms','speedup_vs_serial')}, d['schedule']['profile_t_ns'])"
  done
done
