DBG=0 python tools/gemm_trace.py 2048 1024 1664 128 | sed -n '1p;$p'
python tools/gemm_micro.py 2>&1 | sed -n '7,9p'
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
