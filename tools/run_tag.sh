mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "trap_every_round and 0-" -p no:cacheprovider 2>&1 | tail -2
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "trap or local_search or sigma or caller" -p no:cacheprovider 2>&1 | tail -2
timeout 600 python -m pytest tests/test_gpu_parity_large.py -q -x -k "cfg4_local_search or cfg4_trap_every or cfg4_error_matrix_sigma" -p no:cacheprovider 2>&1 | tail -2
REPS=5 timeout 300 python tools/ls_bench.py 2,3,4 trap 2>&1 | cut -c1-100
timeout 300 python tools/ep_bench.py 5 | tail -1
PM_TRAP_PROF=3 PM_LS_SPARSE=0 PM_MAX_ROUNDS=6 timeout 300 python tools/trap_prof.py 4 | tail -1
