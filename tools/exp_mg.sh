timeout 600 python -m pytest tests -m gpu -x -q -k "branch_placement or chain" 2>&1 | tail -3
timeout 600 python bench.py --config c5 --placement branch --steps 20 --warmup 3 2>&1 | tail -2 | cut -c1-1500
