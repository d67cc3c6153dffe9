#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
timeout 900 python scripts/tune_stencil.py 2>&1 > gpurun_out/tune_stencil_v3.txt
sort -k6 -n gpurun_out/tune_stencil_v3.txt | grep -v BEST | head -12
timeout 900 python bench.py > gpurun_out/bench_v3.json 2> gpurun_out/bench_v3.err; echo bench rc=$?; tail -2 gpurun_out/bench_v3.err; cat gpurun_out/bench_v3.json
