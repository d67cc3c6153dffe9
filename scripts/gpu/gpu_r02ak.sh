#!/bin/bash
# r02ak: xs_lookup pipeline, per-nuclide values by shuffles (1) vs shared-memory broadcast (2)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for M in 9 8; do
  for LG in 0 1; do
    MINB=$M LARGE=$LG AB="-DXS_PIPE=1;-DXS_PIPE=2" timeout 600 python scripts/ab_xs.py 2>&1 | sed "s/^/minB=$M /"
  done
done | tee gpurun_out/ab_xs_pipe_smem_r02ak.txt
