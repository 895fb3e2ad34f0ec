timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "trap or local_search or misaligned or sigma or caller_owned" -p no:cacheprovider 2>&1 | tail -1
timeout 600 python -m pytest tests/test_gpu_parity_large.py -q -x -k "cfg4_local_search or cfg4_trap_every" -p no:cacheprovider 2>&1 | tail -1
REPS=5 timeout 300 python tools/ls_bench.py 2,3,4 trap 2>&1 | cut -c1-100
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -1
