#!/bin/bash
# screen metadata-ring depth variants (BLSH_SX_NM / BLSH_SX_MA), c3 L = 4 at larger W
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02ar_build.log 2>&1
for v in _lib _lib_nm8_ma4 _lib_nm8_ma6 _lib_nm7_ma5 _lib; do
  BLSH_LIB_PATH=$PWD/paper_conf_icde_panm12_b200/$v/libblsh.so timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/r02ar_c4$v.json 2> gpurun_out/r02ar_c4$v.err
  BLSH_TC_MODE=32 BLSH_LIB_PATH=$PWD/paper_conf_icde_panm12_b200/$v/libblsh.so timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 2 > /dev/null 2> gpurun_out/r02ar_tl$v.err
done
for spec in "w341t8:--W 3.41 --T 8" "w341t16:--W 3.41 --T 16"; do
  tag=${spec%%:*}; args=${spec#*:}
  timeout 600 python bench.py --no-cpu-baseline --no-e2e --config c3 --L 4 --hierarchy 0 $args > gpurun_out/r02ar_c3L4_$tag.json 2> gpurun_out/r02ar_c3L4_$tag.err
done
