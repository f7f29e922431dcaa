#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02u_build.log 2>&1
BLSH_TC_MODE=2 ncu --set full --clock-control none --import-source on -k regex:k_screen_f16 -s 1 -c 1 -o gpurun_out/prof_r02u_m2 \
    python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/full_r02u_m2.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_screen_f16 -s 1 -c 1 -o gpurun_out/prof_r02u_m0 \
    python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/full_r02u_m0.log 2>&1
ncu -i gpurun_out/prof_r02u_m2.ncu-rep --page raw --csv > gpurun_out/raw_r02u_m2.csv 2>/dev/null
ncu -i gpurun_out/prof_r02u_m0.ncu-rep --page raw --csv > gpurun_out/raw_r02u_m0.csv 2>/dev/null
