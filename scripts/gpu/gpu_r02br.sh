#!/bin/bash
# scripts/exp_adam_denfold_{noguard,guard}.cu: the r02ax den-folded kernel without and with the r02bf per-block guard (experiment copies, not product)
# r02br: adam_run FOLD=2 (L a factor) vs FOLD=1 (den') under the product's launch bounds
# (minBlocks 5, as W.register sets) and without (ab_adam's default), minBlocks 4/6
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for mb in 5 none 4 6; do
  if [ $mb = none ]; then unset MINB; else export MINB=$mb; fi
  AB="-DADAM_FOLD=1;file:scripts/exp_adam_denfold_noguard.cu;file:scripts/exp_adam_denfold_guard.cu;-DADAM_FOLD=0" timeout 900 python scripts/ab_adam.py 2>&1 | sed "s/^/minB=$mb /" | tee -a gpurun_out/ab_adam_minb_r02br.txt
done
