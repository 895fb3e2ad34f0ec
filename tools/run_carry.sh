mkdir -p gpurun_out
for c in 0 1; do PM_TRAP_CARRY=$c REPS=5 timeout 300 python tools/ls_bench.py 3,4 trap 2>&1 | cut -c1-100; done
PM_TRAP_PROF=3 PM_LS_SPARSE=0 PM_MAX_ROUNDS=6 timeout 300 python tools/trap_prof.py 4 | tail -1
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "trap_every_round" -p no:cacheprovider 2>&1 | tail -1
