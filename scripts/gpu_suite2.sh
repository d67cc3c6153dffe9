#!/bin/bash
# adam_run parity + suite numbers for adam, adam_run, micro, stencil
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "adam" 2>&1 | tail -3
timeout 1800 python bench_suite.py --configs adam,adam_run,micro,stencil > gpurun_out/suite_r01f.jsonl 2> gpurun_out/suite_r01f.err; echo suite rc=$?
tail -3 gpurun_out/suite_r01f.err
for v in jit aot; do timeout 300 python scripts/profile_workloads.py --workload adam_run --variant $v --reps 8 2>&1 | tail -1; done
