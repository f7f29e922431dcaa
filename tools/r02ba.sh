#!/bin/bash
# screen ablations on the final build (BLSH_TC_MODE: 2 no row copies, 4 no MMA, 1 no screen loop; 32 timeline)
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02ba_build.log 2>&1
for m in 0 2 4 1 6; do
  BLSH_TC_MODE=$m timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 3 > gpurun_out/r02ba_c4_m$m.json 2> gpurun_out/r02ba_c4_m$m.err
  BLSH_TC_MODE=$((m+32)) timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 2 > /dev/null 2> gpurun_out/r02ba_tl_m$m.err
done
