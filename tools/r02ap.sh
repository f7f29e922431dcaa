#!/bin/bash
# round measurement batch: smoke, GPU suite, sanitizers, bench lines + oracle arm + launch lists,
# ncu of the screen (traffic on the current sources) and of the warp short-list in the no-reuse regime, shard step
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02ap_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/r02ap_pytest_gpu.log 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_c1.py > gpurun_out/r02ap_san_${tool}.log 2>&1
done
bash tools/round_bench.sh
timeout 900 bash tools/prof.sh full r02ap_screen k_screen_f16
python tools/ncu_summary.py gpurun_out/raw_r02ap_screen.csv > gpurun_out/r02ap_ncu_screen.txt 2>&1
rm -f gpurun_out/prof_r02ap_screen.ncu-rep
for nq in 1000 100000; do
  BLSH_SHORTLIST=warp timeout 900 bash tools/prof.sh full r02ap_warp$nq k_shortlist --config c5 --nq $nq
  python tools/ncu_summary.py gpurun_out/raw_r02ap_warp$nq.csv > gpurun_out/r02ap_ncu_warp$nq.txt 2>&1
  rm -f gpurun_out/prof_r02ap_warp$nq.ncu-rep
done
timeout 900 python tools/shard_step.py --config c4 --world 8 > gpurun_out/r02ap_shard_c4.json 2> gpurun_out/r02ap_shard_c4.err
du -sh gpurun_out
