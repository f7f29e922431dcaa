#!/bin/bash
# TC short-list ablations (debug): prints shortlist ms for BLSH_TC_MODE = 0,1,2,3,4,7
for m in 0 1 2 3 4 7; do
  BLSH_SHORTLIST=tc BLSH_TC_MODE=$m timeout 300 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 1 2>/dev/null \
   | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('mode', $m, 'shortlist_ms', round(d['stage_ms']['ms_shortlist'],2), 'plan_ms', round(d['stage_ms']['ms_plan'],2))"
done
