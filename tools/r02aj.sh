#!/bin/bash
# R33 on the GPU, pipelined API, recalibrated configs: full GPU suite, bench lines c4/c2/c3/c5, p217 calibration
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02aj_build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_pipelined.py tests/test_gpu_e8_recursive.py -q > gpurun_out/r02aj_pytest_new.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/r02aj_pytest_gpu.log 2>&1
timeout 900 python bench.py > gpurun_out/r02aj_bench_c4.json 2> gpurun_out/r02aj_bench_c4.err
for c in c2 c3 c5; do
  timeout 600 python bench.py --no-cpu-baseline --config $c > gpurun_out/r02aj_bench_$c.json 2> gpurun_out/r02aj_bench_$c.err
done
timeout 900 python tools/calibrate.py --config p217 --L 10 --probes 1 --wmult 2.83,4,5.66,8 --out gpurun_out/calib_p217_L10.json > gpurun_out/r02aj_calib_p217.log 2>&1
