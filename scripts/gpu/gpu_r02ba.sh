#!/bin/bash
# r02ba: adam_run -- first float4's loads before the table barrier (ADAM_PREFETCH), and the
# block size (the 977-block grid is 1.32 waves of 5 x 256-thread CTAs per SM); JIT ("all")
# and NVRTC-unfolded ("none") per option, each checked against the fp64 oracle
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
OPTS="-DADAM_PREFETCH=0;-DADAM_PREFETCH=1"
for mode in all none; do
  MODE=$mode AB="$OPTS" timeout 900 python scripts/ab_adam.py 2>&1 | sed "s/^/$mode b256 /" | tee -a gpurun_out/ab_adam_prefetch_r02ba.txt
  MODE=$mode BLOCK=128 MINB=10 AB="$OPTS" timeout 900 python scripts/ab_adam.py 2>&1 | sed "s/^/$mode b128 /" | tee -a gpurun_out/ab_adam_prefetch_r02ba.txt
  MODE=$mode BLOCK=512 MINB=2 AB="$OPTS" timeout 900 python scripts/ab_adam.py 2>&1 | sed "s/^/$mode b512 /" | tee -a gpurun_out/ab_adam_prefetch_r02ba.txt
  MODE=$mode BLOCK=64 MINB=20 AB="$OPTS" timeout 900 python scripts/ab_adam.py 2>&1 | sed "s/^/$mode b64 /" | tee -a gpurun_out/ab_adam_prefetch_r02ba.txt
done
