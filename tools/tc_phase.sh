#!/bin/bash
# TC short-list phase timers under ablation modes (run under gpurun): tools/tc_phase.sh 32 33 ...
for m in "$@"; do
  echo -n "mode $m: "
  BLSH_SHORTLIST=tc BLSH_TC_MODE=$m timeout 300 python bench.py --no-cpu-baseline --no-e2e --steps 1 --warmup 1 2>&1 | grep -E "phase" | tail -1
done
