#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02z_build.log 2>&1
for m in 1 0; do
BLSH_TC_MODE=$m ncu --set full --clock-control none --import-source on -k regex:k_screen_f16 -s 1 -c 1 -o gpurun_out/prof_r02z_m$m \
    python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/full_r02z_m$m.log 2>&1
ncu -i gpurun_out/prof_r02z_m$m.ncu-rep --page raw --csv > gpurun_out/raw_r02z_m$m.csv 2>/dev/null
done
