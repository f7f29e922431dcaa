#!/bin/bash
# round measurement batch on the final sources: smoke, GPU suite, bench lines + oracle arm + launch lists,
# ncu of the screen (traffic on these sources), rescore and probe, small-batch latency, shard step
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02at_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/r02at_pytest_gpu.log 2>&1
bash tools/round_bench.sh
for kre in k_screen_f16 k_tc_rescore k_probe_lookup; do
  timeout 900 bash tools/prof.sh full r02at_$kre $kre
  python tools/ncu_summary.py gpurun_out/raw_r02at_$kre.csv > gpurun_out/r02at_ncu_$kre.txt 2>&1
  rm -f gpurun_out/prof_r02at_$kre.ncu-rep
done
timeout 600 python tools/latency_probe.py --config c5 --batches 1,10,100,1000,10000 > gpurun_out/r02at_latency_c5.jsonl 2> gpurun_out/r02at_latency_c5.err
timeout 900 python tools/shard_step.py --config c4 --world 8 > gpurun_out/r02at_shard_c4.json 2> gpurun_out/r02at_shard_c4.err
du -sh gpurun_out
