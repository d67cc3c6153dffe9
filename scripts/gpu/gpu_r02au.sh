#!/bin/bash
# r02au: xs_lookup XS_PIPE=2 (sentinel-terminated nuclide loop: no trip count on the stack)
# vs XS_PIPE=1, at minBlocks 9 and 8; per-lookup results bit-identical across options
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
AB="-DXS_PIPE=1;-DXS_PIPE=2;-DXS_PIPE=2@8;-DXS_PIPE=1@8" timeout 900 python scripts/ab_xs.py 2>&1 | tee gpurun_out/ab_xs_pipe2_r02au.txt
LARGE=1 AB="-DXS_PIPE=1;-DXS_PIPE=2;-DXS_PIPE=2@8" timeout 900 python scripts/ab_xs.py 2>&1 | tee -a gpurun_out/ab_xs_pipe2_r02au.txt
# r02at's four sanitizer failures: full output per tool, XS alone and everything
for tool in memcheck racecheck; do
  CUDA_CACHE_DISABLE=1 PYTHONPATH=. timeout 900 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize_run.py xs > gpurun_out/san_${tool}_xs_r02au.txt 2>&1; echo san $tool xs rc=$?
  tail -5 gpurun_out/san_${tool}_xs_r02au.txt
done
CUDA_CACHE_DISABLE=1 PYTHONPATH=. timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python scripts/sanitize_run.py > gpurun_out/san_memcheck_all_r02au.txt 2>&1; echo san memcheck all rc=$?
tail -5 gpurun_out/san_memcheck_all_r02au.txt
