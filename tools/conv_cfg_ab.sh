# whole-config A/B: new conv defaults (3 CTAs per SM on 64-channel layers, no halo kernel) vs the
# previous ones (DUET_CONV_OCC=2 DUET_CONV_HALO=1)
for c in c4 c5; do
  for mode in new old new old; do
    if [ $mode = old ]; then export DUET_CONV_OCC=2 DUET_CONV_HALO=1; else unset DUET_CONV_OCC DUET_CONV_HALO; fi
    echo -n "$c $mode: "
    timeout 400 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline --per-config none \
      --tail-samples 200 | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print({k: d.get(k) for k in ('p50_ms','serial_p50_ms','speedup_vs_serial')}, d['schedule']['profile_t_ns'])"
  done
done
