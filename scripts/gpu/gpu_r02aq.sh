#!/bin/bash
# r02aq: final-state validation -- GPU tests, smoke, default bench line
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -4 | tee gpurun_out/r02aq_gpu_tests.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1 | cut -c1-120 | tee gpurun_out/r02aq_smoke.txt
s=$(date +%s); timeout 1500 python bench.py > gpurun_out/bench_r02aq.json 2> gpurun_out/bench_r02aq.err; echo bench rc=$? wall=$(( $(date +%s) - s ))s
