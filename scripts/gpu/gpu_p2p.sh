#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_p2p.py -m gpu -x -q 2>&1 | tail -15
for H in p2p nccl; do
BENCH_SHARE_GPU=1 timeout 400 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr 127.0.0.1 --master-port 29611 bench.py --gpus 2 --steps 50 --warmup 3 --job-sweeps 50 --cpu-seconds 1 --halo $H > gpurun_out/bench_share_$H.json 2> gpurun_out/bench_share_$H.err; echo share $H rc=$?
tail -3 gpurun_out/bench_share_$H.err; cat gpurun_out/bench_share_$H.json
done
