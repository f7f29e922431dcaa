#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02f_build.log 2>&1
bash tools/prof.sh full r02f_screen k_screen_f16
bash tools/prof.sh list r02f_c4
timeout 900 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/r02f_bench_c4.json 2> gpurun_out/r02f_bench_c4.err
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -q -x -k "tc_screen or c4_full_size_properties or c1" > gpurun_out/r02f_pytest.log 2>&1
