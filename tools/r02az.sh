#!/bin/bash
# variant builds: work-item row cap (chr 8k / 32k), k_probe_lookup min blocks (3 / 5); c4 and c3 each
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02az_build.log 2>&1
for v in _lib _lib_chr8k _lib_chr32k _lib_probe3 _lib_probe5; do
  BLSH_LIB_PATH=$PWD/paper_conf_icde_panm12_b200/$v/libblsh.so timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/r02az_c4$v.json 2> gpurun_out/r02az_c4$v.err
  BLSH_LIB_PATH=$PWD/paper_conf_icde_panm12_b200/$v/libblsh.so timeout 600 python bench.py --no-cpu-baseline --no-e2e --config c3 > gpurun_out/r02az_c3$v.json 2> gpurun_out/r02az_c3$v.err
done
