# one-CTA GEMM (M <= 128 rows: MT-DNN encoder, c4's MLP): W on its own issuing warp (default) vs one producer
for r in 1 2; do
  for d in 0 64; do
    for sh in "128 2304 768" "128 3072 768" "128 768 3072" "64 256 512"; do
      DUET_GEMM_DBG=$d timeout 60 python tools/gemm_shape_time.py $sh 10 | sed "s/^/dbg=$d /"
    done
    echo -n "c6 dbg=$d: "; DUET_GEMM_DBG=$d timeout 400 python bench.py --config c6 --steps 100 --warmup 10 --no-cpu-baseline --per-config none --tail-samples 100 | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print({k: d.get(k) for k in ('p50_ms','serial_p50_ms')})"
  done
done
