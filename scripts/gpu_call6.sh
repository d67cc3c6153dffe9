#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -8
timeout 1500 python bench_suite.py > gpurun_out/suite_r01.jsonl 2> gpurun_out/suite_r01.err; echo suite rc=$?
tail -5 gpurun_out/suite_r01.err
cat gpurun_out/suite_r01.jsonl
