#!/bin/bash
# r02bu: final-kernel evidence (after XS_STREAM, XS_SPAN and the final adam_run) -- ncu --set full specialized vs generic for all four
# workload kernels, and the per-workload ablation suite (modes none/lb/rcf/all)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
TAG=r02bu bash scripts/gpu/gpu_spec_vs_generic.sh
timeout 3000 python bench_suite.py --configs adam_run,stencil,xs,xs_large,micro,cache --reps 30 > gpurun_out/suite_r02bu.jsonl 2> gpurun_out/suite_r02bu.err; echo suite rc=$?
