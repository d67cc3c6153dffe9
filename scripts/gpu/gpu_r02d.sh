#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_bench_multirank.py -q -x 2>&1 | tail -15 | tee gpurun_out/r02d_multirank.txt
BLOCKS=128,256 MINBS=1,6,8,9,10,12,16 timeout 900 python scripts/tune_xs_block.py 2>&1 | tee gpurun_out/r02d_tune_xs.txt
