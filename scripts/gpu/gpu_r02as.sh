#!/bin/bash
# r02as: per-block counting sort, out-of-place column scan: tests + timing
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x -k "xs or XS" 2>&1 | tail -15 | tee gpurun_out/r02as_xs_tests.txt
timeout 600 python scripts/xs_step_breakdown.py 2>&1 | tee gpurun_out/xs_step_breakdown_r02as.txt
AB="-DXS_PIPE=1" timeout 600 python scripts/ab_xs.py 2>&1 | tee gpurun_out/ab_xs_sort_r02as.txt
LARGE=1 AB="-DXS_PIPE=1" timeout 600 python scripts/ab_xs.py 2>&1 | tee -a gpurun_out/ab_xs_sort_r02as.txt
