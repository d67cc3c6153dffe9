#!/bin/bash
# r02bs: adam_run with L kept as a factor (R-adam-6 final) at minBlocks 4: Adam GPU tests, the suite's
# Adam line, ncu of adam_run JIT + AOT, the fresh-process e2e jobs at 37 000 and 55 000
# launches (the paper's ADAM AOT range, 2.0-2.9 s)
export PROTEUS_LINEINFO=1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -q -k "adam" 2>&1 | tail -3 | tee gpurun_out/r02bs_tests.txt
for v in jit aot; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:adam_run -s 1 -c 1 -f -o gpurun_out/adam_run_${v}_r02bs python scripts/profile_workloads.py --workload adam_run --variant $v --reps 3 > gpurun_out/prof_adam_run_${v}_r02bs.log 2>&1; echo ncu adam_run $v rc=$?
done
timeout 900 python bench_suite.py --configs adam_run --reps 30 2>&1 | tail -1 | tee gpurun_out/suite_adam_run_r02bs.jsonl
timeout 1500 python bench_suite.py --configs e2e:adam_run@37000 --runs 5 2>&1 | tail -1 | tee gpurun_out/e2e_2s_adam_run_r02bs.jsonl
timeout 1500 python bench_suite.py --configs e2e:adam_run@55000 --runs 5 2>&1 | tail -1 | tee gpurun_out/e2e_adam_run_55k_r02bs.jsonl
