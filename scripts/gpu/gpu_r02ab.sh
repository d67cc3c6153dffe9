#!/bin/bash
# r02ab: short e2e jobs with eager module loading; stencil bench-length job
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 python bench_suite.py --configs e2e:xs,e2e:adam_run,e2e:micro,e2e:stencil --runs 5 > gpurun_out/e2e_short_r02ab.jsonl 2>&1; echo rc=$?
