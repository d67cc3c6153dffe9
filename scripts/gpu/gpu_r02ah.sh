#!/bin/bash
# r02ah: xs_lookup pipeline depth 1 vs 2 at minBlocks 9, 8, 7
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for M in 9 8 7; do
  for LG in 0 1; do
    MINB=$M LARGE=$LG AB="-DXS_PIPE=1;-DXS_PIPE=2" timeout 600 python scripts/ab_xs.py 2>&1 | sed "s/^/minB=$M /"
  done
done | tee gpurun_out/ab_xs_pipe2_r02ah.txt
