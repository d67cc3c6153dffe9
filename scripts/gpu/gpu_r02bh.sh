#!/bin/bash
# r02bh: xs_lookup launch-bounds budget after XS_PACK + XS_CA_LDG: minBlocks 9 (56 regs) vs 10
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
AB="-DXS_CA_LDG=1@9;-DXS_CA_LDG=1@10;-DXS_CA_LDG=1@11" timeout 900 python scripts/ab_xs.py 2>&1 | tee gpurun_out/ab_xs_minb_r02bh.txt
