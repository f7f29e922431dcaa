#!/bin/bash
# warp short-list up to 1 024 queries with few probes; measurement batch on the final sources: GPU suite, smoke + bench lines + oracle arm + launch lists (round_bench.sh),
# ncu of the screen (traffic for these sources), rescore, probe and the warp short-list's no-reuse regime,
# small-batch latency, shard step
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02bf_build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_graph.py -q > gpurun_out/r02bf_pytest_graph.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/r02bf_pytest_gpu.log 2>&1
bash tools/round_bench.sh
for kre in k_screen_f16 k_tc_rescore k_probe_lookup; do
  timeout 900 bash tools/prof.sh full r02bf_$kre $kre
  python tools/ncu_summary.py gpurun_out/raw_r02bf_$kre.csv > gpurun_out/r02bf_ncu_$kre.txt 2>&1
  rm -f gpurun_out/prof_r02bf_$kre.ncu-rep
done
for nq in 1000 100000; do
  BLSH_SHORTLIST=warp timeout 900 bash tools/prof.sh full r02bf_warp$nq k_shortlist --config c5 --nq $nq
  python tools/ncu_summary.py gpurun_out/raw_r02bf_warp$nq.csv > gpurun_out/r02bf_ncu_warp$nq.txt 2>&1
  rm -f gpurun_out/prof_r02bf_warp$nq.ncu-rep
done
timeout 600 python tools/latency_probe.py --config c5 --batches 1,10,100,1000,10000 > gpurun_out/r02bf_latency_c5.jsonl 2> gpurun_out/r02bf_latency_c5.err
timeout 900 python tools/shard_step.py --config c4 --world 8 > gpurun_out/r02bf_shard_c4.json 2> gpurun_out/r02bf_shard_c4.err
timeout 1800 python tools/c5_sweep.py --points multiprobe:8:16,e8_lattice:8:8,morton_curve:8:64 --batches 1,10,100,500,1000,2000,10000,100000 --out gpurun_out/r02bf_c5_batches.jsonl > gpurun_out/r02bf_c5_batches.log 2>&1
