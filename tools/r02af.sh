#!/bin/bash
# shard compaction + shared kk-th screen bound + small-batch dispatch: GPU suite, c4/c3 bench, shard step
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02af_build.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/r02af_pytest_gpu.log 2>&1
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r02af_bench_c4.json 2> gpurun_out/r02af_bench_c4.err
for spec in "c3:--config c3" "c4k50:--config c4 --k 50"; do
  tag=${spec%%:*}; args=${spec#*:}
  timeout 600 python bench.py --no-cpu-baseline --no-e2e $args > gpurun_out/r02af_bench_${tag}.json 2> gpurun_out/r02af_bench_${tag}.err
done
timeout 900 python tools/shard_step.py --config c4 --world 8 > gpurun_out/r02af_shard_c4.json 2> gpurun_out/r02af_shard_c4.err
