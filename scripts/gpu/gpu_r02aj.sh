#!/bin/bash
# r02aj: xs_lookup pipelined (XS_PIPE=1, minBlocks 9): XS GPU tests, ncu of JIT + AOT,
# XS step breakdown, 2 s XS e2e job
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1800 python -m pytest tests -m gpu -q -k "xs or XS" 2>&1 | tail -3 | tee gpurun_out/r02aj_xs_tests.txt
for v in jit aot; do
  R="xs_lookup__jit"; [ $v = aot ] && R="^xs_lookup$"
  timeout 600 ncu --set full --import-source on --clock-control none -k regex:$R -s 1 -c 1 -f -o gpurun_out/xs_${v}_r02aj python scripts/profile_workloads.py --workload xs --variant $v --reps 3 > /dev/null 2>&1; echo ncu xs $v rc=$?
done
timeout 600 python scripts/xs_step_breakdown.py 2>&1 | tee gpurun_out/xs_step_breakdown_r02aj.txt
timeout 900 python bench_suite.py --configs e2e:xs@1500 --runs 5 > gpurun_out/e2e_2s_xs_r02aj.jsonl 2> gpurun_out/e2e_2s_xs_r02aj.err; echo e2e rc=$?
