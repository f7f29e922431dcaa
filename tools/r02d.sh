#!/bin/bash
# Round-2 batch c: fp16 screen with per-item anchor columns.
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02d_build.log 2>&1
for spec in "c1:--config c1 --T 8" "c3:--config c3 --n 200000 --nq 4000 --T 16" "c4:--config c4 --n 2000000 --nq 20000 --T 32"; do
  tag=${spec%%:*}; args=${spec#*:}
  BLSH_TC_DEBUG=/tmp/dbg_$tag.bin timeout 300 python tools/screen_check.py $args > gpurun_out/r02d_check_$tag.log 2>&1
  echo "rc=$?" >> gpurun_out/r02d_check_$tag.log
done
timeout 2400 python -m pytest tests -m gpu -q --maxfail=15 > gpurun_out/r02d_pytest_gpu.log 2>&1
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r02d_bench_c4.json 2> gpurun_out/r02d_bench_c4.err
