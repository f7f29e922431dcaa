#!/bin/bash
# pipelined host-batch API (tests + c4 e2e), c4 W/T recalibration under the fp16 screen, c2 at G = 4 / 8
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02ai_build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_pipelined.py tests/test_abi.py -q > gpurun_out/r02ai_pytest.log 2>&1
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r02ai_bench_c4.json 2> gpurun_out/r02ai_bench_c4.err
timeout 1200 python tools/calibrate.py --config c4 --probes 8,16,32,64 --wmult 4,5.66,8 --out gpurun_out/calib_c4_r02.json > gpurun_out/r02ai_calib_c4.log 2>&1
for G in 4 8; do
  timeout 600 python tools/calibrate.py --config c2 --G $G --probes 1 --wmult 4,8,16,32,64 --out gpurun_out/calib_c2_G${G}_L1.json > gpurun_out/r02ai_calib_c2_G${G}_L1.log 2>&1
  timeout 600 python tools/calibrate.py --config c2 --G $G --L 4 --probes 1 --wmult 4,8,16,32 --out gpurun_out/calib_c2_G${G}_L4.json > gpurun_out/r02ai_calib_c2_G${G}_L4.log 2>&1
done
