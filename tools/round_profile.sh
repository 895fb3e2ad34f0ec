#!/bin/bash
# One GPU session: tests, smoke, bench (ours + reference arm), ncu launch list
# and full captures of the two dominant kernels at the bench workload.
# Usage (from the repo root, via gpurun): tools/round_profile.sh <tag>
tag=${1:-r02}
out=gpurun_out
mkdir -p $out
timeout 1500 python -m pytest tests -m gpu -q --durations=15 -p no:cacheprovider > $out/${tag}_gpu_tests.txt 2>&1; echo "tests rc=$?" >> $out/${tag}_gpu_tests.txt
tail -3 $out/${tag}_gpu_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $out/${tag}_smoke.txt 2>&1; tail -1 $out/${tag}_smoke.txt
timeout 900 python bench.py > $out/${tag}_bench.json 2> $out/${tag}_bench.err; tail -c 300 $out/${tag}_bench.json
timeout 900 python bench.py --impl reference --steps 5 --warmup 1 > $out/${tag}_bench_ref.json 2>&1; tail -c 300 $out/${tag}_bench_ref.json
for c in 2 3; do timeout 600 python bench.py --config $c --no-cpu-baseline > $out/${tag}_bench_cfg$c.json 2>/dev/null; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/${tag}_launches.csv \
  python bench.py --steps 3 --warmup 3 --no-oracle --e2e-steps 1 > /dev/null 2>&1; echo "launch list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k 'regex:k_sad|k_ls_trap' -s 2 -c 2 \
  -o $out/${tag}_full -f python bench.py --steps 1 --warmup 3 --no-oracle --e2e-steps 1 > /dev/null 2>&1; echo "full rc=$?"
