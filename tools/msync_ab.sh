# A/B of the recurrences' step synchronisation: per-128-row-block counters (DUET_RNN_MSYNC=1,
# default) vs one grid barrier (0); single nodes (tools/rnn_time.py) and whole configs (bench.py)
mkdir -p gpurun_out
for m in 1 0 1 0; do
  echo "== DUET_RNN_MSYNC=$m"
  for sh in "gru 4096 1024 256 16" "gru 4096 512 256 32" "lstm 4096 512 256 32" "lstm 4096 256 128 64" \
            "lstm 256 512 256 64" "gru 64 1024 256 64"; do
    DUET_RNN_MSYNC=$m python tools/rnn_time.py $sh
  done
done
for c in ${CONFIGS:-c5 c3}; do
  for m in 1 0; do
    echo "== $c DUET_RNN_MSYNC=$m"
    DUET_RNN_MSYNC=$m timeout 400 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline \
      --per-config none --tail-samples 200 | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print({k: d.get(k) for k in ('p50_ms','serial_p50_ms','speedup_vs_serial')}, d['roofline'] and d['roofline'].get('ms_per_launch'))"
  done
done
