#!/bin/bash
# TRAP: defaults at configs 1-4, thresholds at config 5
out=gpurun_out/$1; mkdir -p $out
REPS=5 timeout 300 python tools/ls_bench.py 1,2,3,4 trap > $out/def.txt 2>&1
for th in 1024 8192 65536; do PM_LS_SPARSE_T=$th REPS=1 timeout 300 python tools/ls_bench.py 5 trap > $out/th5_$th.txt 2>&1; done
