timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "trap or local_search" -p no:cacheprovider 2>&1 | tail -1
timeout 600 python -m pytest tests/test_gpu_parity_large.py -q -x -k "cfg4_local_search or cfg4_trap_every" -p no:cacheprovider 2>&1 | tail -1
REPS=7 timeout 300 python tools/ls_bench.py 3,4 trap 2>&1 | cut -c1-90
