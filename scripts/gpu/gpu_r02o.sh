#!/bin/bash
# r02o: ~2 s e2e jobs with the generic kernels resolved before the clock; default bench line
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 2400 python bench_suite.py --configs e2e:stencil@36000,e2e:adam_run@37000,e2e:xs@1500,e2e:micro@900 --runs 5 > gpurun_out/e2e_2s_r02o.jsonl 2> gpurun_out/e2e_2s_r02o.err; echo e2e2s rc=$?
s=$(date +%s); timeout 1500 python bench.py > gpurun_out/bench_r02o.json 2> gpurun_out/bench_r02o.err; echo bench rc=$? wall=$(( $(date +%s) - s ))s
