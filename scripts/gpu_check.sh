#!/bin/bash
# GPU tests, smoke, the default bench line.
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 900 python bench.py > gpurun_out/bench_chk.json 2> gpurun_out/bench_chk.err; echo bench rc=$?
tail -3 gpurun_out/bench_chk.err; cat gpurun_out/bench_chk.json
