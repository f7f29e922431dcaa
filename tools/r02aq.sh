#!/bin/bash
# route carve-out, sharded-vs-oracle test, e2e gap probe, c3 L = 4 at T = 32
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02aq_build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_pipelined.py -m gpu -q > gpurun_out/r02aq_pytest.log 2>&1
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r02aq_bench_c4.json 2> gpurun_out/r02aq_bench_c4.err
timeout 600 python bench.py --no-cpu-baseline --no-e2e --config c3 --L 4 --hierarchy 0 --T 32 > gpurun_out/r02aq_bench_c3L4.json 2> gpurun_out/r02aq_bench_c3L4.err
timeout 900 python tools/e2e_probe.py --steps 10 > gpurun_out/r02aq_e2e_probe.log 2>&1
timeout 600 bash tools/prof.sh full r02aq_k_route k_route
python tools/ncu_summary.py gpurun_out/raw_r02aq_k_route.csv > gpurun_out/r02aq_ncu_k_route.txt 2>&1
rm -f gpurun_out/prof_r02aq_k_route.ncu-rep
