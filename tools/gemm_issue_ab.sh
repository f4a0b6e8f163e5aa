# pair GEMM: A and W on separate issuing warps (default) vs one producer (DUET_GEMM_DBG=64)
for r in 1 2; do
  for d in 0 64; do
    for sh in "2048 1024 1664" "2048 512 1024" "2048 256 512" "4096 1024 1664" "4096 2048 512" "4096 1024 2048" "8192 8192 8192"; do
      DUET_GEMM_DBG=$d python tools/gemm_shape_time.py $sh 10 | sed "s/^/dbg=$d /"
    done
  done
done
for d in 0 64 0 64; do
  echo -n "c2 dbg=$d: "; DUET_GEMM_DBG=$d timeout 300 python bench.py --config c2 --steps 200 --warmup 10 --no-cpu-baseline --per-config none --tail-samples 200 | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print({k: d.get(k) for k in ('p50_ms','serial_p50_ms','speedup_vs_serial')}, d['roofline']['ms_per_launch'], d['roofline']['frac'])"
done
