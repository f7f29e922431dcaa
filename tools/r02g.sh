#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02g_build.log 2>&1
for m in 0 64; do
  BLSH_TC_MODE=$m timeout 900 python bench.py --no-cpu-baseline --no-e2e --steps 3 > gpurun_out/r02g_bench_m$m.json 2> gpurun_out/r02g_bench_m$m.err
done
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -q -x -k "tc_screen or c4_full_size_properties or c1" > gpurun_out/r02g_pytest.log 2>&1
