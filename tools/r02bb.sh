#!/bin/bash
# source-line attribution of the final k_screen_f16 and k_probe_lookup (ncu source page, gzipped)
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02bb_build.log 2>&1
for kre in k_screen_f16 k_probe_lookup k_tc_rescore; do
  timeout 900 bash tools/prof.sh full r02bb_$kre $kre
  ncu -i gpurun_out/prof_r02bb_$kre.ncu-rep --page source --csv > gpurun_out/src_r02bb_$kre.csv 2>/dev/null
  gzip -f gpurun_out/src_r02bb_$kre.csv
  rm -f gpurun_out/prof_r02bb_$kre.ncu-rep gpurun_out/raw_r02bb_$kre.csv
done
ls -la gpurun_out
