#!/bin/bash
# TC short-list ablations (debug): prints shortlist ms for BLSH_TC_MODE values (default 0 1 2 3 4 7).
# bits: 1 skip screen, 2 zero-fill row loads, 4 skip MMA, 64 skip A stores to TMEM, 128 skip staging copies
modes=${@:-0 1 2 3 4 7}
for m in $modes; do
  BLSH_SHORTLIST=tc BLSH_TC_MODE=$m timeout 300 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 1 2>/dev/null \
   | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('mode', $m, 'shortlist_ms', round(d['stage_ms']['ms_shortlist'],2), 'screen_ms', round(d['stage_ms']['ms_screen'],2))"
done
