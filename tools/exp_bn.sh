for bn in 64 128; do for c in c3 c4; do DUET_RNN_BN=$bn timeout 400 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bn_${c}_$bn.log 2>&1; done; done
