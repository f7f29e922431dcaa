#!/bin/bash
# R31/R32 + KT=64 screen parity; ground truth for c2/c3/c5/p217; C5 sweep; c3 recalibration
mkdir -p gpurun_out/bench_data
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02ae_build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_curve.py tests/test_gpu_parity.py -m gpu -q -x > gpurun_out/r02ae_pytest.log 2>&1
for c in c2 c3 c5 p217; do
  timeout 600 python tools/make_gt.py --config $c --sample 1000 --out-dir gpurun_out/bench_data > gpurun_out/r02ae_gt_$c.log 2>&1
  cp gpurun_out/bench_data/${c}_gt.npz bench_data/ 2>/dev/null
done
timeout 1200 python tools/c5_sweep.py --out gpurun_out/c5_sweep.jsonl > gpurun_out/r02ae_c5_sweep.log 2>&1
timeout 900 python tools/calibrate.py --config c3 --G 8 --hier --probes 1,4,8,16,32 --wmult 2.83,4,5.66 --out gpurun_out/calib_c3_G8.json > gpurun_out/r02ae_calib_c3_G8.log 2>&1
timeout 900 python tools/calibrate.py --config c3 --G 4 --hier --probes 1,4,8,16,32 --wmult 2.83,4,5.66 --out gpurun_out/calib_c3_G4.json > gpurun_out/r02ae_calib_c3_G4.log 2>&1
for spec in "c3:--config c3" "c2:--config c2" "c4k50:--config c4 --k 50"; do
  tag=${spec%%:*}; args=${spec#*:}
  timeout 600 python bench.py --no-cpu-baseline $args > gpurun_out/r02ae_bench_${tag}.json 2> gpurun_out/r02ae_bench_${tag}.err
done
