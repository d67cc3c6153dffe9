#!/bin/bash
# r02bp: adam_run ADAM_FOLD=2 (L = lr/bc1 kept as a factor: no division by L, always finite,
# no per-block guard -- the generic build back at 48 registers) vs ADAM_FOLD=1 (den' folded +
# guard: 56 registers in the generic build); specialized and NVRTC-unfolded per option
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for mode in all none; do
  MODE=$mode AB="-DADAM_FOLD=1;-DADAM_FOLD=2;-DADAM_FOLD=2 -DADAM_RCP_SPLIT=2" timeout 900 python scripts/ab_adam.py 2>&1 | sed "s/^/$mode /" | tee -a gpurun_out/ab_adam_fold2_r02bp.txt
done
