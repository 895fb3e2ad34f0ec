mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "sigma or caller or photomosaic or error_matrix" -p no:cacheprovider 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_parity_large.py -q -x -k "cfg4_error_matrix_sigma or cfg4_photomosaic" -p no:cacheprovider 2>&1 | tail -2
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/sig_bench.json 2> gpurun_out/sig_bench.err; tail -c 600 gpurun_out/sig_bench.json
