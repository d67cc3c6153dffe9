#!/bin/bash
# r02 baseline check: GPU tests + bench line on the round-1 build.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
timeout 900 python bench.py > gpurun_out/bench_r02a.json 2> gpurun_out/bench_r02a.err; echo bench rc=$?
tail -3 gpurun_out/bench_r02a.err; cat gpurun_out/bench_r02a.json | head -c 3000
