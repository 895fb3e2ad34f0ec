#!/bin/bash
# One GPU session: tests, smoke, bench, ncu launch lists and full captures.
# Usage (from the repo root, via gpurun): tools/round_profile.sh <tag>
tag=${1:-r01}
out=gpurun_out
mkdir -p $out
timeout 1200 python -m pytest tests -m gpu -q -x > $out/${tag}_gpu_tests.txt 2>&1; echo "tests rc=$?" >> $out/${tag}_gpu_tests.txt
tail -3 $out/${tag}_gpu_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $out/${tag}_smoke.txt 2>&1; tail -1 $out/${tag}_smoke.txt
timeout 600 python bench.py > $out/${tag}_bench.json 2> $out/${tag}_bench.err; tail -1 $out/${tag}_bench.json
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $out/${tag}_bench_ref.json 2>&1; tail -1 $out/${tag}_bench_ref.json
# launch list, kernel nodes (graph-launched kernels inside conditional bodies are not listed in this mode)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/${tag}_launches.csv \
  python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1; echo "launch list rc=$?"
# launch list with every CUDA-graph launch as one workload (the sparse-round graph appears as a row)
timeout 600 ncu --graph-profiling graph --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file $out/${tag}_launches_graph.csv \
  python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1; echo "graph launch list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k 'regex:k_sad|k_ls_trap' -s 2 -c 2 \
  -o $out/${tag}_full -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1; echo "full rc=$?"
timeout 900 ncu --graph-profiling graph --set full --clock-control none -s 1 -c 1 --kernel-name-base function \
  -o $out/${tag}_sparse_graph -f python tools/ls_bench.py 2 trap > /dev/null 2>&1; echo "sparse graph full rc=$?"
REPS=3 timeout 600 python tools/assign_bench.py 1 2 3 4 > $out/${tag}_assign.txt 2>&1; tail -4 $out/${tag}_assign.txt
REPS=3 timeout 900 python tools/ls_bench.py 1,2 trap,window,walk,cta,class > $out/${tag}_ls_methods.txt 2>&1
REPS=2 timeout 900 python tools/ls_bench.py 3 auto,trap,walk,class,cta >> $out/${tag}_ls_methods.txt 2>&1
REPS=1 timeout 900 python tools/ls_bench.py 4 auto,class >> $out/${tag}_ls_methods.txt 2>&1; grep cfg $out/${tag}_ls_methods.txt | cut -c1-90
timeout 600 python tools/e_bench.py 1,2,3,4,5 > $out/${tag}_e_bench.txt 2>&1; cat $out/${tag}_e_bench.txt | grep cfg
