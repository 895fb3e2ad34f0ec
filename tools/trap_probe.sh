#!/bin/bash
out=gpurun_out/$1; mkdir -p $out
timeout 900 python -m pytest tests -x -q -m gpu -k "trap or local_search or photomosaic" > $out/pytest.log 2>&1; echo rc=$? >> $out/pytest.log
PM_TRAP_CLUSTER=0 PM_LS_SPARSE=0 timeout 120 python tools/trap_prof.py 2,3 > $out/prof.txt 2>&1
REPS=5 timeout 300 python tools/ls_bench.py 1,2,3,4 trap > $out/ls.txt 2>&1
PM_TRAP_NBSYNC=0 REPS=5 timeout 300 python tools/ls_bench.py 3,4 trap > $out/ls_nonb.txt 2>&1
REPS=1 timeout 600 python tools/ls_bench.py 5 trap > $out/ls5.txt 2>&1
