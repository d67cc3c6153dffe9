#!/bin/bash
# r02j: phases of the short adam_run e2e jobs (async outliers), bench default run (suite with XS minBlocks 9)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python bench_suite.py --configs e2e:adam_run --runs 8 > gpurun_out/e2e_adam_phases_r02j.jsonl 2>&1; echo rc=$?
timeout 1500 python bench.py > gpurun_out/bench_r02j.json 2> gpurun_out/bench_r02j.err; echo bench rc=$?
