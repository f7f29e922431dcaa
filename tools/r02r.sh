#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02r_build.log 2>&1
BLSH_BUILD_DIR=/tmp/blsh_spin BLSH_NVCC_FLAGS=-DBLSH_SPIN_WAIT=1 python -m paper_conf_icde_panm12_b200.build --force >> gpurun_out/r02r_build.log 2>&1
for v in base spin; do
  lib=""; [ $v = spin ] && lib=/tmp/blsh_spin/libblsh.so
  for m in 32 39; do
    BLSH_LIB_PATH=$lib BLSH_TC_MODE=$m timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 2 --warmup 1 > gpurun_out/r02r_${v}_m$m.json 2> gpurun_out/r02r_${v}_m$m.err
    echo "$v mode $m" >> gpurun_out/r02r_summary.txt; grep "\[tc\] per item" gpurun_out/r02r_${v}_m$m.err | tail -1 >> gpurun_out/r02r_summary.txt
    python -c "import json; d=json.loads(open('gpurun_out/r02r_${v}_m$m.json').read().strip().splitlines()[-1]); print('screen', round(d['stage_ms']['ms_screen'],3), 'total', round(d['stage_ms']['ms_total'],3))" >> gpurun_out/r02r_summary.txt
  done
done
