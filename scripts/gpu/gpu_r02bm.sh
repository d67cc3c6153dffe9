#!/bin/bash
# r02bm: xs_lookup XS_SPAN -- warps of one material spanning up to 1 + XS_SPAN energy bins
# (the ~15% of warps that straddle a sort-bucket boundary) take the shuffle path on the
# union bracket instead of the per-lane bisection; bit-identical per lookup
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
AB="-DXS_SPAN=0;-DXS_SPAN=1;-DXS_SPAN=3" timeout 900 python scripts/ab_xs.py 2>&1 | tee gpurun_out/ab_xs_span_r02bm.txt
LARGE=1 AB="-DXS_SPAN=0;-DXS_SPAN=1;-DXS_SPAN=3" timeout 900 python scripts/ab_xs.py 2>&1 | tee -a gpurun_out/ab_xs_span_r02bm.txt
