# GPU box: N3 model-variation parity tests and the §VI-D sweeps (Figs. 14-17).
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "seq_output or variation" -s > gpurun_out/n3_tests.log 2>&1; echo tests_rc=$? >> gpurun_out/n3_tests.log
timeout 1500 python tools/sweeps.py --out gpurun_out/sweeps.json > gpurun_out/sweeps.log 2>&1; echo sweeps_rc=$? >> gpurun_out/sweeps.log
