#!/bin/bash
# c3 screen-overflow experiment (BLSH_SCAPW), route/hash staging ablation, ncu of the non-screen c4 kernels
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02ak_build.log 2>&1
for sc in 96 192 384; do
  BLSH_TC_MODE=0 BLSH_SCAPW=$sc timeout 600 python bench.py --no-cpu-baseline --no-e2e --config c3 > gpurun_out/r02ak_c3_scap$sc.json 2> gpurun_out/r02ak_c3_scap$sc.err
done
BLSH_RH_STAGE=1 timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/r02ak_c4_rhstage.json 2> gpurun_out/r02ak_c4_rhstage.err
for kre in k_route k_hash k_expand_atoms k_probe_lookup k_tc_rescore k_tile_prep; do
  timeout 600 bash tools/prof.sh full r02ak_$kre "$kre"
  python tools/ncu_summary.py gpurun_out/raw_r02ak_$kre.csv > gpurun_out/r02ak_ncu_$kre.txt 2>&1
  ncu -i gpurun_out/prof_r02ak_$kre.ncu-rep --page source --csv > gpurun_out/src_r02ak_$kre.csv 2>/dev/null; rm -f gpurun_out/prof_r02ak_$kre.ncu-rep
done
