timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_assign.py tests/test_gpu_histogram.py -q -x -k "error_matrix or sigma or pack or photomosaic or paper_grid or sad or assignment or render" -p no:cacheprovider 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity_large.py -q -x -k "error_matrix" -p no:cacheprovider 2>&1 | tail -1
timeout 600 python tools/e_bench.py 1,2,3,4,5 2>&1 | grep "cfg"
