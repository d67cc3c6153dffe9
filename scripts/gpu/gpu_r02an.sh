#!/bin/bash
# r02an: ptxas optimisation level for the specializations: compile ms and kernel time
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
CUDA_CACHE_DISABLE=1 AB=";-Xptxas=-O1;-Xptxas=-O2" timeout 1200 python scripts/ab_nvrtc_opts.py 2>&1 | tee gpurun_out/ab_ptxas_opt_r02an.txt
