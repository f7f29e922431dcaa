#!/bin/bash
# re-validate the restored build: GPU suite, smoke, c4 bench, launch list, ncu of the screen
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02ad_build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r02ad_pytest_gpu.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02ad_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/r02ad_bench_c4.json 2> gpurun_out/r02ad_bench_c4.err
timeout 600 bash tools/prof.sh list r02ad_c4
timeout 900 bash tools/prof.sh full r02ad_screen k_screen_f16
python tools/ncu_summary.py gpurun_out/raw_r02ad_screen.csv > gpurun_out/r02ad_ncu_screen.txt 2>&1
