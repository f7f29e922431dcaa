#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02j_build.log 2>&1
for m in 32 33 39; do
  BLSH_TC_MODE=$m timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 2 --warmup 1 > gpurun_out/r02j_m$m.json 2> gpurun_out/r02j_m$m.err
  echo "mode $m" >> gpurun_out/r02j_summary.txt; grep "\[tc\]" gpurun_out/r02j_m$m.err | tail -2 >> gpurun_out/r02j_summary.txt
done
