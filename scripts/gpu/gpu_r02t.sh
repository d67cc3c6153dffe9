#!/bin/bash
# r02t: the per-workload ablation suite (modes none/lb/rcf/all, registers, in-process e2e) on the r02 build
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 3000 python bench_suite.py --configs adam_run,stencil,xs,xs_large,micro,cache --reps 30 > gpurun_out/suite_r02t.jsonl 2> gpurun_out/suite_r02t.err; echo rc=$?
