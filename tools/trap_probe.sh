#!/bin/bash
# TRAP development probe: parity tests, then whole-search timings (sparse hand-over on)
out=gpurun_out/$1; mkdir -p $out
timeout 900 python -m pytest tests -x -q -m gpu -k "trap or local_search or photomosaic" > $out/pytest.log 2>&1; echo rc=$? >> $out/pytest.log
REPS=5 timeout 300 python tools/ls_bench.py 1,2,3,4 trap,window,class > $out/ls.txt 2>&1
PM_TRAP_CLUSTER=0 REPS=5 timeout 300 python tools/ls_bench.py 1,2,3 trap > $out/ls_grid.txt 2>&1
for v in 1 2 3; do PM_TRAP_V=$v REPS=5 timeout 300 python tools/ls_bench.py 1,2,3,4 trap > $out/ls_v$v.txt 2>&1; done
