#!/bin/bash
# r02m: the default bench line, wall time
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
s=$(date +%s); timeout 1500 python bench.py > gpurun_out/bench_r02m.json 2> gpurun_out/bench_r02m.err; echo bench rc=$? wall=$(( $(date +%s) - s ))s
