#!/bin/bash
# r02ag: xs_lookup software-pipelined bracket loads (XS_PIPE) A/B at minBlocks 9 and 8
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for M in 9 8; do
  for LG in 0 1; do
    MINB=$M LARGE=$LG AB="-DXS_PIPE=0;-DXS_PIPE=1" timeout 600 python scripts/ab_xs.py 2>&1 | sed "s/^/minB=$M /"
  done
done | tee gpurun_out/ab_xs_pipe_r02ag.txt
