#!/bin/bash
# r02y: xs_lookup result staging off/on (event order either way)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python scripts/ab_xs.py 2>&1 | tee gpurun_out/r02y_ab_xs_stage.txt
LARGE=1 timeout 900 python scripts/ab_xs.py 2>&1 | tee -a gpurun_out/r02y_ab_xs_stage.txt
