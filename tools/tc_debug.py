"""Check the tensor-core screen's dot products against numpy (debug aid).

    BLSH_TC_DEBUG=/tmp/tcdbg.bin python tools/tc_debug.py
Runs one C1-sized query through the library with the TC short-list, then
compares the TMEM dot products of work item 0 / block 0 with float64 numpy.
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
from paper_conf_icde_panm12_b200 import blsh  # noqa: E402

path = os.environ.setdefault("BLSH_TC_DEBUG", "/tmp/tcdbg.bin")
cfg = synth.CONFIGS["c1"]
X, Q = synth.make_dataset(cfg)
ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=4, M=8, W=4.0, seed=21)
ids, d2, nc = ix.query(torch.from_numpy(Q).cuda(), 10, probe=1, n_probes=16)
torch.cuda.synchronize()
st = ix.stats()
print("tiled", st.tiled, "total_cand", st.total_cand, "rescored", st.pairs_scored, "union", st.union_rows)
raw = np.fromfile(path, dtype=np.float32)
dots = raw[:4096].reshape(128, 32)
xn = raw[4096:4096 + 128]
rpos = raw[4096 + 128:4096 + 256].view(np.uint32)
msk = raw[4096 + 256:4096 + 384].view(np.uint32)
qn = raw[4096 + 384:4096 + 416]
qord = np.fromfile(path, dtype=np.uint32)[4096 + 512:4096 + 512 + 32]
perm = ix.export("PERM")
Xp = X[perm]
nqt = int((qn > 0).sum())                     # tile 0's queries (qn = 0 for empty slots)
c = Q[qord[:nqt]].astype(np.float64).mean(0)  # tile centre = mean of its queries
qs = Q[qord].astype(np.float64) - c
qs[nqt:] = 0.0
valid = msk != 0
xs = Xp[rpos].astype(np.float64) - c
ref = xs @ qs.T
err = np.abs(dots - ref)[valid]
print("rows valid", valid.sum(), "max |dot err|", err.max(), "max |dot|", np.abs(ref[valid]).max())
print("xn err", np.abs(xn - (xs ** 2).sum(1))[valid].max(), "qn err", np.abs(qn - (qs ** 2).sum(1)).max())
print("sample dots", dots[0, :4], ref[0, :4])
# which (row, column) of the reference best explains each measured dot row (layout probe)
for r in range(3):
    best = [(float(np.abs(dots[r] - ref[rr]).max()), rr) for rr in range(128) if valid[rr]]
    print("row", r, "closest ref row", min(best))
