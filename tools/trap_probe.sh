#!/bin/bash
out=gpurun_out/$1; mkdir -p $out
timeout 900 python -m pytest tests -x -q -m gpu -k "trap or local_search or photomosaic or multi_rank" > $out/pytest.log 2>&1; echo rc=$? >> $out/pytest.log
PM_LS_SPARSE=0 timeout 120 python tools/trap_prof.py 1,2,3 > $out/prof.txt 2>&1
PM_TRAP_EP=0 PM_LS_SPARSE=0 timeout 120 python tools/trap_prof.py 1,2,3 > $out/prof_noep.txt 2>&1
REPS=5 timeout 300 python tools/ls_bench.py 1,2,3,4 trap > $out/ls.txt 2>&1
