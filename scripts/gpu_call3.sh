#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -25
timeout 600 python scripts/tune_stencil.py 2>&1 | tail -200 > gpurun_out/tune_stencil_r01.txt
tail -3 gpurun_out/tune_stencil_r01.txt
