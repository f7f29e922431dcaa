#!/bin/bash
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02aa_build.log 2>&1
for m in 32 33 34; do
  BLSH_TC_MODE=$m timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 2 --warmup 1 > gpurun_out/r02aa_m$m.json 2> gpurun_out/r02aa_m$m.err
  echo "mode $m" >> gpurun_out/r02aa_summary.txt; grep "\[tc\] per item" gpurun_out/r02aa_m$m.err | tail -1 >> gpurun_out/r02aa_summary.txt
  python -c "import json; d=json.loads(open('gpurun_out/r02aa_m$m.json').read().strip().splitlines()[-1]); print('screen', round(d['stage_ms']['ms_screen'],3), 'total', round(d['stage_ms']['ms_total'],3))" >> gpurun_out/r02aa_summary.txt
done
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "tc_screen or c1" > gpurun_out/r02aa_pytest.log 2>&1
