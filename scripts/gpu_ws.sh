#!/bin/bash
mkdir -p gpurun_out
CONFIGS="4,2,6;4,2,8;5,2,6;6,2,6;7,2,6;2,4,6;2,4,8;3,4,6;4,4,6;3,3,6;5,3,6;4,3,6;2,3,8;8,2,5;6,1,8;5,1,10" ZCS="2,3,4,5,6,8" EXTRA="-DWS_L2HINT=1" timeout 1200 python scripts/tune_stencil_ws.py > gpurun_out/tune_ws_wide.txt 2>&1; echo tune rc=$?
tail -1 gpurun_out/tune_ws_wide.txt
