#!/bin/bash
# One GPU session: tests, smoke, bench, ncu launch list and full captures.
# Usage (from the repo root, via gpurun): tools/round_profile.sh <tag>
tag=${1:-r01}
out=gpurun_out
mkdir -p $out
timeout 1200 python -m pytest tests -m gpu -q -x > $out/${tag}_gpu_tests.txt 2>&1; echo "tests rc=$?" >> $out/${tag}_gpu_tests.txt
tail -3 $out/${tag}_gpu_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $out/${tag}_smoke.txt 2>&1; tail -1 $out/${tag}_smoke.txt
timeout 600 python bench.py > $out/${tag}_bench.json 2> $out/${tag}_bench.err; tail -1 $out/${tag}_bench.json
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $out/${tag}_bench_ref.json 2>&1; tail -1 $out/${tag}_bench_ref.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/${tag}_launches.csv \
  python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1; echo "launch list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k 'regex:k_sad|k_ls_window|k_sp_' -s 4 -c 4 \
  -o $out/${tag}_full -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1; echo "full rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k 'regex:k_auction' -c 1 \
  -o $out/${tag}_auction -f python tools/assign_bench.py 2 > /dev/null 2>&1; echo "auction full rc=$?"
REPS=3 timeout 600 python tools/assign_bench.py 1 2 3 4 > $out/${tag}_assign.txt 2>&1; tail -4 $out/${tag}_assign.txt
