#!/bin/bash
# micro_column warp-per-column + rain gating: parity, sanitizers, suite line, ncu jit/aot.
export PROTEUS_LINEINFO=1
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "micro or sanitizer or edge" 2>&1 | tail -3
timeout 900 python bench_suite.py --configs micro > gpurun_out/suite_micro_r01h.jsonl 2> gpurun_out/suite_micro_r01h.err; echo suite rc=$?
for v in jit aot; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:micro_column -s 2 -c 1 -f -o gpurun_out/sg_micro_${v}_r01i python scripts/profile_workloads.py --workload micro --variant $v --reps 3 > /dev/null 2>&1; echo ncu micro $v rc=$?
done
