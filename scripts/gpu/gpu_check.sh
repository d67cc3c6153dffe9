#!/bin/bash
# GPU tests, smoke, native hit latency, the default bench line
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1 | cut -c1-200
bash scripts/gpu/gpu_hitlat.sh 2>&1 | tail -3
timeout 900 python bench.py > gpurun_out/bench_chk.json 2> gpurun_out/bench_chk.err; echo bench rc=$?
tail -3 gpurun_out/bench_chk.err; cat gpurun_out/bench_chk.json
