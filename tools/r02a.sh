#!/bin/bash
# Round-2 first GPU batch: 1000-query c4 ground truth, GPU suite, c4 bench, ncu captures, sanitizers.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r02a_smi.txt 2>&1
nproc > gpurun_out/r02a_nproc.txt
( time timeout 1200 python tools/make_gt.py --config c4 --sample 1000 ) > gpurun_out/r02a_gt.log 2>&1
cp bench_data/c4_gt.npz gpurun_out/c4_gt.npz
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/r02a_pytest_gpu.log 2>&1
timeout 900 python bench.py > gpurun_out/r02a_bench_c4.json 2> gpurun_out/r02a_bench_c4.err
bash tools/prof.sh full r02a_tc k_shortlist_tc
bash tools/prof.sh full r02a_hash "k_hash<"
ncu --set full --clock-control none --import-source on -k regex:k_hash_rows -s 0 -c 1 -o gpurun_out/prof_r02a_hashrows \
    python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/full_r02a_hashrows.log 2>&1
ncu -i gpurun_out/prof_r02a_hashrows.ncu-rep --page raw --csv > gpurun_out/raw_r02a_hashrows.csv 2>/dev/null
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_c1.py > gpurun_out/r02a_san_${tool}.log 2>&1
done
