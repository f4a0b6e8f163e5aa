#!/bin/bash
# ncu --set full captures of the round-2 fp32 (3xTF32) kernels and the tcgen05 attention (GPU box)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
full() {  # name regex skip cmd...
  local name=$1 rx=$2 skip=$3; shift 3
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"$rx" -s $skip -c 1 \
      -o gpurun_out/${name}_r2 "$@" > gpurun_out/ncu_${name}_r2.log 2>&1
  ncu -i gpurun_out/${name}_r2.ncu-rep --page raw --csv > gpurun_out/${name}_r2_raw.csv 2>/dev/null
}
full fc1_f32 "gemm_tf32x3" 2 python tools/gemm_micro_one.py 2048 1024 1664 f32
full conv_l3_f32 "gemm_tf32x3" 2 python tools/gemm_micro_one.py conv 64 14 14 256 256 3 1 1 f32
full conv_l3_bf16 "conv_tma" 2 python tools/gemm_micro_one.py conv 64 14 14 256 256 3 1 1
python tools/full_md2.py r2_tf32 --no-summary fc1_f32=gpurun_out/fc1_f32_r2_raw.csv \
    conv_l3_f32=gpurun_out/conv_l3_f32_r2_raw.csv conv_l3_bf16=gpurun_out/conv_l3_bf16_r2_raw.csv
cp profiles/r2_tf32_full.md gpurun_out/ 2>/dev/null
