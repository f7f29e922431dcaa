#!/bin/bash
# route without prefetch + streaming row loads, rescore back to 4 rows, sync-free small batches,
# screen ring released in slot pairs: GPU suite, c4 bench + per-item timeline, small-batch latency, ncu
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02an_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r02an_pytest_gpu.log 2>&1
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r02an_bench_c4.json 2> gpurun_out/r02an_bench_c4.err
BLSH_TC_MODE=32 timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 2 > gpurun_out/r02an_c4_timeline.json 2> gpurun_out/r02an_c4_timeline.err
timeout 900 python tools/c5_sweep.py --points multiprobe:8:16,e8_lattice:8:8 --batches 1,10,100,1000,10000 --out gpurun_out/r02an_c5_batches.jsonl > gpurun_out/r02an_c5_batches.log 2>&1
for kre in k_route k_hash k_tc_rescore; do
  timeout 600 bash tools/prof.sh full r02an_$kre "$kre"
  python tools/ncu_summary.py gpurun_out/raw_r02an_$kre.csv > gpurun_out/r02an_ncu_$kre.txt 2>&1
  rm -f gpurun_out/prof_r02an_$kre.ncu-rep
done
timeout 600 ncu --set full --clock-control none -k regex:k_hash_rows -c 1 -o gpurun_out/prof_r02an_hash_rows \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/full_r02an_hash_rows.log 2>&1
ncu -i gpurun_out/prof_r02an_hash_rows.ncu-rep --page raw --csv > gpurun_out/raw_r02an_hash_rows.csv 2>/dev/null
python tools/ncu_summary.py gpurun_out/raw_r02an_hash_rows.csv > gpurun_out/r02an_ncu_k_hash_rows.txt 2>&1
rm -f gpurun_out/prof_r02an_hash_rows.ncu-rep
