#!/bin/bash
# r02s: micro e2e (~2 s job) after the r02p/r02r kernel changes
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 python bench_suite.py --configs e2e:micro@1000 --runs 5 > gpurun_out/e2e_2s_micro_r02s.jsonl 2>&1; echo rc=$?
