# GPU round trip: tests, benches with the measured gate-tile choice, sweeps, ncu round evidence.
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q -s > gpurun_out/t2_tests.log 2>&1; echo tests_rc=$? >> gpurun_out/t2_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/t2_smoke.log 2>&1
timeout 300 python bench.py > gpurun_out/t2_bench_c2.log 2>&1
for c in c1 c3 c4 c5 c6; do timeout 600 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/t2_bench_$c.log 2>&1; done
timeout 1500 python tools/sweeps.py --out gpurun_out/sweeps_t2.json > gpurun_out/sweeps_t2.log 2>&1; echo sweeps_rc=$? >> gpurun_out/sweeps_t2.log
bash tools/ncu_round.sh r1d
