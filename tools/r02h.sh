#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02h_build.log 2>&1
for m in 0 1 2 3 4 7; do
  BLSH_TC_MODE=$m timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 2 > gpurun_out/r02h_m$m.json 2> gpurun_out/r02h_m$m.err
  python -c "import json; d=json.loads(open('gpurun_out/r02h_m$m.json').read().strip().splitlines()[-1]); print('mode $m', round(d['stage_ms']['ms_screen'],3), round(d['stage_ms']['ms_total'],3))" >> gpurun_out/r02h_summary.txt
done
