#!/bin/bash
# compute-sanitizer over the round-2 kernels (tools/sanitize_run.py); one line per run
run() { # name, env..., tool
  local name=$1; shift; local tool=$1; shift
  out=$(env "$@" timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_run.py 2>&1)
  rc=$?; summ=$(echo "$out" | grep -E "ERROR SUMMARY|RACECHECK SUMMARY|sanitize workload ok" | tr '\n' ' ')
  echo "$name | $tool | rc=$rc | $summ"
}
for tool in memcheck racecheck synccheck; do
  run "auto (TRAP 128x32 cluster+grid, sparse Ep scan, cwalk16)" $tool METHODS=trap
  run "TRAP 192x48 grid, spec always, no sparse" $tool METHODS=trap PM_TRAP_V=6 PM_TRAP_SPEC=2 PM_LS_SPARSE=0
  run "TRAP 128x32 grid, per-thread staging" $tool METHODS=trap PM_TRAP_V=5 PM_TRAP_CLUSTER=0 PM_TRAP_COAL=0
  run "TRAP from E rows (no Ep)" $tool METHODS=trap PM_TRAP_EP=0
  run "multi-rank emulated x2 (192x48)" $tool METHODS=trap MULTI=2 PM_TRAP_V=6
  run "walk (cwalk 16) + window + class" $tool METHODS=walk,window,class PM_LS_CWALK=1
  run "E split-K 64x2 + 128x3" $tool METHODS=class PM_SAD_PLAN=64002
done
