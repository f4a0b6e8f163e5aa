#!/bin/bash
# stem kernel phase isolation (DUET_STEM_DBG: 1 skip build, 2 skip MMA, 4 skip stores, 8 skip patch
# TMA), c4 and c5 stem shapes, CUDA-graph timing.  Output: gpurun_out/stem_dbg.log
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
: > gpurun_out/stem_dbg.log
for shape in "64 224 3 64 7 2 3" "4096 32 3 64 7 2 3"; do
  for d in 0 1 2 4 8 5 13 15; do
    echo "dbg $d: $(DUET_STEM_DBG=$d CONV_ONE_GRAPH=1 python tools/conv_one.py $shape 10 2>&1 | tail -1)" >> gpurun_out/stem_dbg.log
  done
done
cat gpurun_out/stem_dbg.log
