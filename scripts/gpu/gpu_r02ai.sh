#!/bin/bash
# r02ai: xs_lookup pipeline variants (1: bracket ahead; 3: + f from the bracket, records
# without E; conc as a uniform load) at minBlocks 9 and 8 (variants 3 and CONC_LOAD since removed)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for M in 9 8; do
  for LG in 0 1; do
    MINB=$M LARGE=$LG AB="-DXS_PIPE=1;-DXS_PIPE=3;-DXS_PIPE=1 -DXS_PIPE_CONC_LOAD=1" timeout 600 python scripts/ab_xs.py 2>&1 | sed "s/^/minB=$M /"
  done
done | tee gpurun_out/ab_xs_pipe3_r02ai.txt
