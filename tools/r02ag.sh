#!/bin/bash
# large-k TC path, kk-rule for KT >= 32: GPU suite, shard step breakdown, c3 recalibration, k = 500
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02ag_build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/r02ag_pytest_gpu.log 2>&1
timeout 900 python tools/shard_step.py --config c4 --world 8 > gpurun_out/r02ag_shard_c4.json 2> gpurun_out/r02ag_shard_c4.err
for spec in "c3k500:--config c3 --k 500" "c3G8k500:--config c3 --G 8 --k 500" "c4:--config c4"; do
  tag=${spec%%:*}; args=${spec#*:}
  timeout 600 python bench.py --no-cpu-baseline --no-e2e $args > gpurun_out/r02ag_bench_${tag}.json 2> gpurun_out/r02ag_bench_${tag}.err
done
timeout 900 python tools/calibrate.py --config c3 --G 8 --hier --probes 4,8,16,32 --wmult 4,5.66,8 --out gpurun_out/calib_c3_G8b.json > gpurun_out/r02ag_calib_c3_G8.log 2>&1
timeout 900 python tools/calibrate.py --config c3 --G 8 --probes 8,16,32,64 --wmult 5.66,8,11.3 --out gpurun_out/calib_c3_G8_nohier.json > gpurun_out/r02ag_calib_c3_G8_nohier.log 2>&1
