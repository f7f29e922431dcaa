#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02ac_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/r02ac_pytest_gpu.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02ac_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/r02ac_bench_c4.json 2> gpurun_out/r02ac_bench_c4.err
