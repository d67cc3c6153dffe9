#!/bin/bash
# r02bb: xs_lookup XS_PACK (bracket start + width in one shuffled word: one SHFL per nuclide
# fewer) vs the shipped loop, minBlocks 9 and 8; per-lookup results bit-identical
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
AB="-DXS_PACK=0;-DXS_PACK=1;-DXS_PACK=1@8" timeout 900 python scripts/ab_xs.py 2>&1 | tee gpurun_out/ab_xs_pack_r02bb.txt
LARGE=1 AB="-DXS_PACK=0;-DXS_PACK=1" timeout 900 python scripts/ab_xs.py 2>&1 | tee -a gpurun_out/ab_xs_pack_r02bb.txt
