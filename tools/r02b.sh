#!/bin/bash
# Round-2 batch b: bring-up of the fp16 compact-table screen.
mkdir -p gpurun_out
python -m paper_conf_icde_panm12_b200.build > gpurun_out/r02b_build.log 2>&1
BLSH_TC_DEBUG=/tmp/dbg1.bin timeout 180 python tools/screen_check.py --config c1 --T 8 > gpurun_out/r02b_check_c1.log 2>&1
echo "rc=$?" >> gpurun_out/r02b_check_c1.log
BLSH_TC_DEBUG=/tmp/dbg3.bin timeout 300 python tools/screen_check.py --config c3 --n 200000 --nq 4000 --T 16 > gpurun_out/r02b_check_c3.log 2>&1
echo "rc=$?" >> gpurun_out/r02b_check_c3.log
timeout 300 python - > gpurun_out/r02b_nonfinite_dbg.log 2>&1 <<'PY'
import numpy as np, torch, synth
from paper_conf_icde_panm12_b200 import blsh
X, Q = synth.make_dataset(synth.CONFIGS["c1"])
Q = Q.copy(); Q[3, 0] = np.nan; Q[7, 5] = np.inf
ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=4, M=8, W=4.0, seed=42, keep_stages=True)
ix.query(torch.from_numpy(Q).cuda(), 10, probe=1, n_probes=16, keep_stages=True)
torch.cuda.synchronize()
print("lib", blsh.LIB_PATH)
print("oor", ix.export("Q_OOR")[:10])
print("t", ix.export("Q_T").reshape(-1, 8)[[3, 7]])
PY
timeout 2400 python -m pytest tests -m gpu -q --maxfail=15 > gpurun_out/r02b_pytest_gpu.log 2>&1
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r02b_bench_c4.json 2> gpurun_out/r02b_bench_c4.err
BLSH_SCREEN=tf32 timeout 900 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/r02b_bench_c4_tf32.json 2>&1
