mkdir -p gpurun_out
for c in c4 c5; do timeout 600 python tools/node_times.py $c > gpurun_out/nodes_$c.log 2>&1; done
CONFIGS="c1 c3 c4 c5" bash tools/run_all.sh
