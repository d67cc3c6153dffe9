#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "adam" 2>&1 | tail -2
for v in jit aot; do timeout 300 python scripts/profile_workloads.py --workload adam_run --variant $v --reps 8 2>&1 | tail -1; done
