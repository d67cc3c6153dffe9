#!/bin/bash
# r02bk: xs_lookup L2 hints -- XS_STREAM=1: perm read and results written evict-first
# (__ldcs/__stcs) so the 440 MB of outputs do not evict the 43 MB table; =2: + the table
# reads of the pipelined loop with an L2 evict_last policy; bit-identical per lookup
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
AB="-DXS_STREAM=0;-DXS_STREAM=1;-DXS_STREAM=2" timeout 900 python scripts/ab_xs.py 2>&1 | tee gpurun_out/ab_xs_stream_r02bk.txt
LARGE=1 AB="-DXS_STREAM=0;-DXS_STREAM=1;-DXS_STREAM=2" timeout 900 python scripts/ab_xs.py 2>&1 | tee -a gpurun_out/ab_xs_stream_r02bk.txt
