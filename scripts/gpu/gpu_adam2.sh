#!/bin/bash
# Adam with reciprocal / SFU arithmetic (R-adam-5): parity + timing + ncu of adam_run.
export PROTEUS_LINEINFO=1   # ncu --import-source maps JIT kernels to their source
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "adam" 2>&1 | tail -4
for v in jit aot; do
  timeout 300 python scripts/profile_workloads.py --workload adam_run --variant $v --reps 8 2>&1 | tail -1
  timeout 300 python scripts/profile_workloads.py --workload adam --variant $v --reps 8 2>&1 | tail -1
done
timeout 600 python bench_suite.py --configs adam,adam_run > gpurun_out/suite_adam2.jsonl 2> gpurun_out/suite_adam2.err; echo suite rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:adam_run -s 1 -c 1 -f -o gpurun_out/adam_run_jit_r01h python scripts/profile_workloads.py --workload adam_run --variant jit --reps 3 > /dev/null 2>&1; echo ncu rc=$?
