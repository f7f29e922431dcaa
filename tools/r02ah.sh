#!/bin/bash
# session 3 re-validation of HEAD: GPU suite (no -x), smoke, c4 bench + launch list + ncu of the screen,
# shard step, c3 (G = 8) and c2 calibration
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02ah_build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r02ah_pytest_gpu.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02ah_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/r02ah_bench_c4.json 2> gpurun_out/r02ah_bench_c4.err
timeout 600 bash tools/prof.sh list r02ah_c4
timeout 900 bash tools/prof.sh full r02ah_screen k_screen_f16
python tools/ncu_summary.py gpurun_out/raw_r02ah_screen.csv > gpurun_out/r02ah_ncu_screen.txt 2>&1
timeout 600 python tools/shard_step.py --config c4 --world 8 > gpurun_out/r02ah_shard_c4.json 2> gpurun_out/r02ah_shard_c4.err
timeout 900 python tools/calibrate.py --config c3 --G 8 --hier --probes 8,16,32 --wmult 4,5.66,8 --out gpurun_out/calib_c3_G8h.json > gpurun_out/r02ah_calib_c3_G8h.log 2>&1
timeout 600 python tools/calibrate.py --config c2 --probes 1 --wmult 4,8,16,32,64 --out gpurun_out/calib_c2_L1.json > gpurun_out/r02ah_calib_c2_L1.log 2>&1
timeout 600 python tools/calibrate.py --config c2 --L 8 --probes 1 --wmult 2,4,8,16 --out gpurun_out/calib_c2_L8.json > gpurun_out/r02ah_calib_c2_L8.log 2>&1
