#!/bin/bash
# Profiling helper (run under gpurun).  Usage:
#   tools/prof.sh list <tag> [bench args...]          launch list of the timed region (ncu, NVTX "timed")
#   tools/prof.sh full <tag> <kernel-regex> [bench args...]   ncu --set full of one launch of a kernel
set -u
mode=$1; tag=$2; shift 2
mkdir -p gpurun_out
if [ "$mode" = "list" ]; then
  ncu --metrics gpu__time_duration.sum --clock-control none --nvtx --nvtx-include "timed/" --csv \
      --log-file gpurun_out/launches_${tag}.csv \
      python bench.py --steps 2 --warmup 1 --nvtx --no-cpu-baseline --no-e2e "$@" > gpurun_out/list_${tag}.log 2>&1
else
  kre=$1; shift
  ncu --set full --clock-control none --import-source on -k regex:${kre} -s 1 -c 1 -o gpurun_out/prof_${tag} \
      python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e "$@" > gpurun_out/full_${tag}.log 2>&1
  ncu -i gpurun_out/prof_${tag}.ncu-rep --page raw --csv > gpurun_out/raw_${tag}.csv 2>/dev/null
fi
