#!/bin/bash
# chunk-staged route/hash kernels, single-pass k_expand_atoms, scap 384 for k > 16: GPU suite + c4/c3 bench + ncu of route/hash/expand
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02al_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r02al_pytest_gpu.log 2>&1
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r02al_bench_c4.json 2> gpurun_out/r02al_bench_c4.err
timeout 600 python bench.py --no-cpu-baseline --no-e2e --config c3 > gpurun_out/r02al_bench_c3.json 2> gpurun_out/r02al_bench_c3.err
for kre in k_route k_hash k_expand_atoms; do
  timeout 600 bash tools/prof.sh full r02al_$kre "$kre"
  python tools/ncu_summary.py gpurun_out/raw_r02al_$kre.csv > gpurun_out/r02al_ncu_$kre.txt 2>&1
  rm -f gpurun_out/prof_r02al_$kre.ncu-rep
done
