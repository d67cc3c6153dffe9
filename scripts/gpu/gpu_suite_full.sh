#!/bin/bash
# full suite refresh (CFG 1-5) + GPU tests
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 2400 python bench_suite.py > gpurun_out/suite_r01g.jsonl 2> gpurun_out/suite_r01g.err; echo suite rc=$?
tail -3 gpurun_out/suite_r01g.err
