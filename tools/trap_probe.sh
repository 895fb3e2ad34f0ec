#!/bin/bash
out=gpurun_out/$1; mkdir -p $out
timeout 900 python -m pytest tests -x -q -m gpu -k "trap or local_search" > $out/pytest.log 2>&1; echo rc=$? >> $out/pytest.log
REPS=5 timeout 300 python tools/ls_bench.py 1,2,3,4 trap > $out/ls.txt 2>&1
REPS=1 timeout 600 python tools/ls_bench.py 5 trap > $out/ls5.txt 2>&1
