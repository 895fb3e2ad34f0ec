mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "caller_owned or trap_every_round" -p no:cacheprovider 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_parity_large.py -q -x -k "cfg4_caller or cfg4_local_search" -p no:cacheprovider 2>&1 | tail -2
timeout 300 python tools/ep_bench.py 5
