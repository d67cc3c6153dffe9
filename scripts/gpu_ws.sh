#!/bin/bash
mkdir -p gpurun_out
for U in 1 5 10; do
MINB=4 CONFIGS="4,2,6;4,2,8;7,1,8" ZCS="3,4" EXTRA="-DWS_UNROLL=$U" timeout 900 python scripts/tune_stencil_ws.py > gpurun_out/tune_ws_u$U.txt 2>&1; echo unroll $U; grep -v BEST gpurun_out/tune_ws_u$U.txt
done
