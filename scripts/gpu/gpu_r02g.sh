#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do
BLOCKS=128,256 MINBS=4,6,8,9,10 timeout 900 python scripts/tune_xs_block.py 2>&1 | tee -a gpurun_out/r02g_tune_xs.txt
done
