#!/bin/bash
# cp.async row staging in k_tc_rescore / k_tc_emit / k_shortlist: GPU suite, bench lines, ncu
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02au_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r02au_pytest_gpu.log 2>&1
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r02au_bench_c4.json 2> gpurun_out/r02au_bench_c4.err
for spec in "p217:--config p217" "c3k500:--config c3 --k 500" "c3e8h:--config c3 --quantizer 1 --probe 2 --T 16 --hierarchy 1" "c5L4:--config c5 --L 4 --T 4" "c2:--config c2"; do
  tag=${spec%%:*}; args=${spec#*:}
  timeout 600 python bench.py --no-cpu-baseline --no-e2e $args > gpurun_out/r02au_bench_${tag}.json 2> gpurun_out/r02au_bench_${tag}.err
done
timeout 900 bash tools/prof.sh full r02au_rescore k_tc_rescore
python tools/ncu_summary.py gpurun_out/raw_r02au_rescore.csv > gpurun_out/r02au_ncu_rescore.txt 2>&1
rm -f gpurun_out/prof_r02au_rescore.ncu-rep
for nq in 1000 100000; do
  BLSH_SHORTLIST=warp timeout 900 bash tools/prof.sh full r02au_warp$nq k_shortlist --config c5 --nq $nq
  python tools/ncu_summary.py gpurun_out/raw_r02au_warp$nq.csv > gpurun_out/r02au_ncu_warp$nq.txt 2>&1
  rm -f gpurun_out/prof_r02au_warp$nq.ncu-rep
done
timeout 600 python tools/latency_probe.py --config c5 --batches 1,10,100,1000 > gpurun_out/r02au_latency_c5.jsonl 2> gpurun_out/r02au_latency_c5.err
