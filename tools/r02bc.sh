#!/bin/bash
# rescore: next pair batch prefetched; GPU suite, c4/c3/c5 bench, ncu of the rescore
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02bc_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r02bc_pytest_gpu.log 2>&1
for c in c4 c3 c5; do
  timeout 600 python bench.py --no-cpu-baseline --no-e2e --config $c > gpurun_out/r02bc_bench_$c.json 2> gpurun_out/r02bc_bench_$c.err
done
timeout 900 bash tools/prof.sh full r02bc_rescore k_tc_rescore
python tools/ncu_summary.py gpurun_out/raw_r02bc_rescore.csv > gpurun_out/r02bc_ncu_rescore.txt 2>&1
rm -f gpurun_out/prof_r02bc_rescore.ncu-rep
