#!/bin/bash
# r01h: edge tests, the CFG 1-5 suite, the default bench line.
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_edge.py -x -q 2>&1 | tail -3
timeout 2400 python bench_suite.py > gpurun_out/suite_r01h.jsonl 2> gpurun_out/suite_r01h.err; echo suite rc=$?
tail -3 gpurun_out/suite_r01h.err
timeout 900 python bench.py > gpurun_out/bench_r01h2.json 2> gpurun_out/bench_r01h2.err; echo bench rc=$?
cat gpurun_out/bench_r01h2.json
