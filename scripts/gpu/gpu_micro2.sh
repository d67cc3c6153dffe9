#!/bin/bash
# micro_column: exhaustive div_fast check, parity, minBlocks sweep, jit/aot timing
mkdir -p gpurun_out
timeout 600 python scripts/exp_div_fast.py 2>&1 | tee gpurun_out/div_fast_exhaustive.txt | tail -4
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "micro or spec_routines" 2>&1 | tail -3
timeout 900 python scripts/tune_min_blocks.py micro 2>&1 | tee gpurun_out/tune_micro_minb.txt | tail -9
for v in jit aot; do timeout 300 python scripts/profile_workloads.py --workload micro --variant $v --reps 8 2>&1 | tail -1; done
