mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "trap_every_round or speculative" -p no:cacheprovider 2>&1 | tail -2
for v in 6 7; do PM_TRAP_V=$v REPS=3 timeout 300 python tools/ls_bench.py 4,5 trap 2>&1 | cut -c1-120; done
timeout 300 python tools/ep_bench.py 5
PM_TRAP_PROF=3 PM_LS_SPARSE=0 PM_MAX_ROUNDS=4 timeout 300 python tools/trap_prof.py 5 | tail -1
