#!/bin/bash
# GPU suite after the small-batch/route changes; c4 bench; small-batch latency; the f-row lines at the new configs; shard step
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02ao_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r02ao_pytest_gpu.log 2>&1
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r02ao_bench_c4.json 2> gpurun_out/r02ao_bench_c4.err
timeout 900 python tools/c5_sweep.py --points multiprobe:8:16,e8_lattice:8:8 --batches 1,10,100,1000 --out gpurun_out/r02ao_c5_batches.jsonl > gpurun_out/r02ao_c5_batches.log 2>&1
for spec in "p217:--config p217" "c3k500:--config c3 --k 500" "c3e8h:--config c3 --quantizer 1 --probe 2 --T 16 --hierarchy 1" \
            "c5curve:--config c5 --probe 3 --T 64" "c3L4:--config c3 --L 4 --hierarchy 0 --T 8" "c2:--config c2" "c5:--config c5"; do
  tag=${spec%%:*}; args=${spec#*:}
  timeout 600 python bench.py --no-cpu-baseline --no-e2e $args > gpurun_out/r02ao_bench_${tag}.json 2> gpurun_out/r02ao_bench_${tag}.err
done
timeout 900 python tools/shard_step.py --config c4 --world 8 > gpurun_out/r02ao_shard_c4.json 2> gpurun_out/r02ao_shard_c4.err
