#!/bin/bash
# r02az: adam_run (folded) -- part of the sqrt on the FMA pipe (ADAM_SQRT_SPLIT) to unload
# the SFU, and the time-loop unroll factor; specialized ("all") and NVRTC-unfolded ("none",
# the generic build's stand-in) per option, each checked against the fp64 oracle
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
OPTS="-DADAM_SQRT_SPLIT=0;-DADAM_SQRT_SPLIT=1;-DADAM_SQRT_SPLIT=1 -DADAM_RCP_SPLIT=0;-DADAM_SQRT_SPLIT=2 -DADAM_RCP_SPLIT=0;-DADAM_SQRT_SPLIT=1 -DADAM_RCP_SPLIT=2;-DADAM_UNROLL=4;-DADAM_UNROLL=4 -DADAM_SQRT_SPLIT=1;-DADAM_UNROLL=1"
for mode in all none; do
  MODE=$mode AB="$OPTS" timeout 900 python scripts/ab_adam.py 2>&1 | sed "s/^/$mode /" | tee -a gpurun_out/ab_adam_sqrt_r02az.txt
done
