mkdir -p gpurun_out
# the multi-rank bench flow (torchrun, 2 ranks, max-over-ranks timing) on a one-GPU box: gloo, both ranks on GPU 0
DUET_DIST_BACKEND=gloo DUET_FORCE_DEVICE=0 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29531 bench.py --gpus 2 --steps 20 --warmup 3 > gpurun_out/ranks2.log 2>&1; echo rc=$? >> gpurun_out/ranks2.log
DUET_DIST_BACKEND=gloo DUET_FORCE_DEVICE=0 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29532 bench.py --impl reference --gpus 2 --steps 2 --warmup 1 > gpurun_out/ranks2_ref.log 2>&1; echo rc=$? >> gpurun_out/ranks2_ref.log
