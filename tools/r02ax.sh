#!/bin/bash
# tile-cut threshold sweep (BLSH_TILE_JUMP) on c4 and c3
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02ax_build.log 2>&1
for j in 64 128 512 2048 8192; do
  BLSH_TILE_JUMP=$j timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/r02ax_c4_j$j.json 2> gpurun_out/r02ax_c4_j$j.err
  BLSH_TILE_JUMP=$j timeout 600 python bench.py --no-cpu-baseline --no-e2e --config c3 > gpurun_out/r02ax_c3_j$j.json 2> gpurun_out/r02ax_c3_j$j.err
done
