#!/bin/bash
# r02aw/ax: adam_run with the step-uniform factors folded (ADAM_FOLD: 6 instead of 8 FMA-pipe
# instructions per element-step) vs the shipped form, SFU/FMA reciprocal split re-tuned;
# each variant checked against the fp64 oracle (1e-5)
mkdir -p gpurun_out  # r02ax (TAG=r02ax): den-folded form, one rounding of p per step
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
AB="-DADAM_FOLD=0;-DADAM_FOLD=1;-DADAM_FOLD=1 -DADAM_RCP_SPLIT=0;-DADAM_FOLD=1 -DADAM_RCP_SPLIT=1;-DADAM_FOLD=1 -DADAM_RCP_SPLIT=3" timeout 900 python scripts/ab_adam.py 2>&1 | tee gpurun_out/ab_adam_fold_${TAG:-r02aw}.txt
MINB=6 AB="-DADAM_FOLD=1;-DADAM_FOLD=1 -DADAM_RCP_SPLIT=1" timeout 900 python scripts/ab_adam.py 2>&1 | sed 's/^/minB6 /' | tee -a gpurun_out/ab_adam_fold_${TAG:-r02aw}.txt
MINB=4 AB="-DADAM_FOLD=1;-DADAM_FOLD=1 -DADAM_RCP_SPLIT=1" timeout 900 python scripts/ab_adam.py 2>&1 | sed 's/^/minB4 /' | tee -a gpurun_out/ab_adam_fold_${TAG:-r02aw}.txt
