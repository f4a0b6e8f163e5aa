for dbg in 0 2; do
  echo "=== DBG=$dbg"
  DBG=$dbg python tools/gemm_trace.py 2048 1024 1664 128 | sed -n '1p;$p'
  DBG=$dbg python tools/gemm_trace.py 2048 1024 1664 256 | sed -n '$p'
done
python tools/gemm_micro.py
