#!/bin/bash
# r02ar: per-block counting sort for the XS step (xs_bin/xs_scan/xs_scatter, column scan in place): tests + timing
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x -k "xs or XS" 2>&1 | tail -15 | tee gpurun_out/r02ar_xs_tests.txt
timeout 600 python scripts/xs_step_breakdown.py 2>&1 | tee gpurun_out/xs_step_breakdown_r02ar.txt
AB="-DXS_PIPE=1" timeout 600 python scripts/ab_xs.py 2>&1 | tee gpurun_out/ab_xs_sort_r02ar.txt
LARGE=1 AB="-DXS_PIPE=1" timeout 600 python scripts/ab_xs.py 2>&1 | tee -a gpurun_out/ab_xs_sort_r02ar.txt
