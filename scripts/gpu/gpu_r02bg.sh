#!/bin/bash
# r02bg: xs_lookup XS_CA_LDG (the concentration loaded per nuclide as a warp-uniform load
# instead of a 64-bit shuffle: no LDL/STL left in the SASS at minBlocks 9) vs the shipped
# loop; per-lookup results bit-identical
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
AB="-DXS_CA_LDG=0;-DXS_CA_LDG=1;-DXS_CA_LDG=1@8" timeout 900 python scripts/ab_xs.py 2>&1 | tee gpurun_out/ab_xs_caldg_r02bg.txt
LARGE=1 AB="-DXS_CA_LDG=0;-DXS_CA_LDG=1" timeout 900 python scripts/ab_xs.py 2>&1 | tee -a gpurun_out/ab_xs_caldg_r02bg.txt
