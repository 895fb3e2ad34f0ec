#!/bin/bash
# Sweep the auction's eps schedule, Gauss-Seidel tail threshold, pair keeping
# and shared-memory prices (env knobs read by k_assign.cu).
export PM_AUCTION_DEBUG=1
for keep in ${KEEPS:-1 0}; do for gs in ${GSS:-0 4 16 64 256}; do for th in ${THS:-4 8}; do for sh in ${SHS:-3 4}; do
  PM_AUCTION_KEEP=$keep PM_AUCTION_GS=$gs PM_AUCTION_THETA=$th PM_AUCTION_EPS_SHIFT=$sh REPS=2 timeout 120 python tools/assign_bench.py ${CFGS:-2 3}
done; done; done; done
