#!/bin/bash
# r02bx: the XS energy-bin count (index + sort key) re-measured on the final lookup kernel
# (multi-bin shuffle path, packed bracket word, streaming stores): 2048 / 4096 / 8192
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
AB="2048,4096,8192" timeout 1500 python scripts/ab_xs_ebins.py 2>&1 | tee gpurun_out/ab_xs_ebins_r02bx.txt
