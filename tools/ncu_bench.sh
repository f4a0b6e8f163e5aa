# ncu evidence for the bench workload (c2).  Usage on the GPU box: bash tools/ncu_bench.sh <tag>
TAG=${1:-r1}
mkdir -p gpurun_out
# 1) launch list of our kernels during 3 timed steps (cold-cache, serialised: compare shares)
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    -k regex:"gemm|gather|hash|join|conv|im2col|pool|mlp|rnn|reduce|add_act|sigmoid|logit|concat" --csv --log-file gpurun_out/launches_${TAG}.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu-baseline --profile-samples 2 > gpurun_out/ncu_launch_${TAG}.log 2>&1
# 2) full profile of the dominant kernel (fc1 = the first gemm2 launch with grid y = 8)
ncu --set full --clock-control none --import-source on -k regex:gemm2_kernel -s 6 -c 3 \
    -o gpurun_out/fc1_${TAG} python bench.py --steps 1 --warmup 1 --no-cpu-baseline --profile-samples 2 \
    > gpurun_out/ncu_full_${TAG}.log 2>&1
ncu -i gpurun_out/fc1_${TAG}.ncu-rep --page raw --csv > gpurun_out/fc1_${TAG}_raw.csv 2>/dev/null
