#!/bin/bash
# r02u: the default bench (e2e jobs on) under torchrun with 2 and 4 ranks sharing the GPU
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for N in 2 4; do
BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $N --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus $N --steps 200 --warmup 5 > gpurun_out/bench_share_n${N}_r02u.json 2> gpurun_out/bench_share_n${N}_r02u.err; echo N=$N rc=$?
tail -c 600 gpurun_out/bench_share_n${N}_r02u.json
grep "\[bench\]" gpurun_out/bench_share_n${N}_r02u.err | head -3
done
