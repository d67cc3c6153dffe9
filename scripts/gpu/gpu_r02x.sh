#!/bin/bash
# r02x: XS e2e after the fairness fix (xs_index generic in every variant, tables before the clock)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 python bench_suite.py --configs e2e:xs,e2e:adam_run,e2e:micro --runs 5 > gpurun_out/e2e_short_r02x.jsonl 2>&1; echo rc=$?
