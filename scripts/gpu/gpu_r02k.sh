#!/bin/bash
# r02k: stencil4_ws L2 priorities A/B (WS_L2HINT 1 vs 3) over z-chunk counts
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do
for H in 1 4; do
echo "== WS_L2HINT=$H rep $rep" | tee -a gpurun_out/r02k2_l2hint.txt
EXTRA="-DWS_L2HINT=$H" CONFIGS="4,2,6" ZCS="4,8" timeout 600 python scripts/tune_stencil_ws.py 2>&1 | grep -v BEST | tee -a gpurun_out/r02k2_l2hint.txt
done; done
