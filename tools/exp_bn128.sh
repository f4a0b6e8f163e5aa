{
python tools/rnn_time.py gru 64 1024 256 64
DUET_RNN_BN=128 python tools/rnn_time.py gru 64 1024 256 64
python tools/rnn_time.py lstm 256 512 256 64
DUET_RNN_BN=128 python tools/rnn_time.py lstm 256 512 256 64
} > gpurun_out/exp_bn128.log 2>&1
for c in c3 c4; do
timeout 300 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_bn64_$c.log 2>&1
DUET_RNN_BN=128 timeout 300 python bench.py --config $c --steps 100 --warmup 10 --no-cpu-baseline > gpurun_out/bench_bn128_$c.log 2>&1
done
