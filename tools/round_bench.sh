#!/bin/bash
# Round-end measurement batch (run under gpurun): the headline bench line, the
# next-row workloads, the oracle arm and launch lists.  Output in gpurun_out/.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/rb_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/rb_c4.json 2> gpurun_out/rb_c4.err
for spec in "p217:--config p217" "c3k500:--config c3 --k 500" "c3e8h:--config c3 --quantizer 1 --probe 2 --T 16 --hierarchy 1" \
            "c5curve:--config c5 --probe 3 --T 64" "c5L4:--config c5 --L 4 --T 4" "c3:--config c3" "c2:--config c2" "c5:--config c5"; do
  tag=${spec%%:*}; args=${spec#*:}
  timeout 600 python bench.py --no-cpu-baseline $args > gpurun_out/rb_${tag}.json 2> gpurun_out/rb_${tag}.err
done
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/rb_ref.json 2> gpurun_out/rb_ref.err
bash tools/prof.sh list c4
bash tools/prof.sh list p217 --config p217
bash tools/prof.sh list c3e8h --config c3 --quantizer 1 --probe 2 --T 16 --hierarchy 1
