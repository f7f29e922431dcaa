#!/bin/bash
# C5 sweep on the final build: probes 1-64 x three families x W, batch 1-100k at each family's best point
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02be_build.log 2>&1
timeout 3000 python tools/c5_sweep.py --out gpurun_out/c5_sweep_final.jsonl > gpurun_out/r02be_c5_sweep.log 2>&1
