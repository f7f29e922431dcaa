#!/bin/bash
# grouped route passes (k_route_pass), screen metadata ring 8: GPU suite, c4 bench, c5 L = 4 lines, ncu of the route
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02as_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r02as_pytest_gpu.log 2>&1
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r02as_bench_c4.json 2> gpurun_out/r02as_bench_c4.err
for spec in "c5L4t4:--config c5 --L 4 --T 4" "c5L4t8:--config c5 --L 4 --T 8" "c3:--config c3" "c5:--config c5"; do
  tag=${spec%%:*}; args=${spec#*:}
  timeout 600 python bench.py --no-cpu-baseline --no-e2e $args > gpurun_out/r02as_bench_${tag}.json 2> gpurun_out/r02as_bench_${tag}.err
done
timeout 600 bash tools/prof.sh full r02as_route k_route_pass
python tools/ncu_summary.py gpurun_out/raw_r02as_route.csv > gpurun_out/r02as_ncu_route.txt 2>&1
rm -f gpurun_out/prof_r02as_route.ncu-rep
timeout 600 python tools/shard_step.py --config c4 --world 8 > gpurun_out/r02as_shard_c4.json 2> gpurun_out/r02as_shard_c4.err
