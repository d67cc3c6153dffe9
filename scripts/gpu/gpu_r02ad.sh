#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python scripts/exp_bench_kernel_only.py 2>&1 | tee gpurun_out/r02ad.txt
