#!/bin/bash
# prefetched chunk staging (route/hash/hash_rows), atom-parallel k_expand_atoms, rescore 8 rows in flight
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02am_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r02am_pytest_gpu.log 2>&1
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r02am_bench_c4.json 2> gpurun_out/r02am_bench_c4.err
timeout 600 python bench.py --no-cpu-baseline --no-e2e --config c3 > gpurun_out/r02am_bench_c3.json 2> gpurun_out/r02am_bench_c3.err
for kre in k_route k_hash k_expand_atoms k_tc_rescore k_hash_rows; do
  timeout 600 bash tools/prof.sh full r02am_$kre "$kre"
  python tools/ncu_summary.py gpurun_out/raw_r02am_$kre.csv > gpurun_out/r02am_ncu_$kre.txt 2>&1
  rm -f gpurun_out/prof_r02am_$kre.ncu-rep
done
