mkdir -p gpurun_out
(REPS=2 timeout 600 python tools/ls_bench.py 5 trap; timeout 600 python tools/sp_rounds.py 5 trap | cut -c1-140; PM_TRAP_PROF=3 PM_LS_SPARSE=0 PM_MAX_ROUNDS=12 timeout 600 python tools/trap_prof.py 5 | tail -1) > gpurun_out/sp5.txt 2>&1
cat gpurun_out/sp5.txt
