"""Check the fp16 screen's first block against numpy (bring-up / layout check).

    BLSH_TC_DEBUG=/tmp/dbg.bin python tools/screen_check.py [--config c1] [--n N] [--nq NQ]

Runs one query batch through the tensor-core screen with the debug dump on (item 0,
block 0: per row the 32 query dots, the two centre dots, beta, m, E, table row, mask,
K slot, |s r|, s_b; eta per query; S, S_c, C_c, nqt), then recomputes in numpy fp64,
for every (row, query) pair of the block whose mask bit is set:
  exact d2 = |q_j - x|^2, the screen's d~2 = K_aj + beta_i + m_i D_ij with K_aj from
  numpy, and checks lo <= d2 <= up (the screen's rigorous bound) and reports the
  bound width relative to d2.
"""
from __future__ import annotations

import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c1")
    ap.add_argument("--n", type=int, default=None)
    ap.add_argument("--nq", type=int, default=None)
    ap.add_argument("--T", type=int, default=8)
    a = ap.parse_args()
    import torch
    import synth
    from paper_conf_icde_panm12_b200 import blsh
    path = os.environ.get("BLSH_TC_DEBUG")
    assert path, "set BLSH_TC_DEBUG"
    cfg = synth.CONFIGS[a.config]
    X, Q = synth.make_dataset(cfg, n=a.n, nq=a.nq, backend="torch", device="cuda")
    ix = blsh.blsh_build(X, n_leaves=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index)
    ids, d2, nc = ix.query(Q, 10, probe=1 if a.T > 1 else 0, n_probes=a.T)
    torch.cuda.synchronize()
    print("tiled kind", ix.stats().tiled)
    raw = np.fromfile(path, dtype=np.uint8)
    h = raw[: (4096 + 2048) * 4].view(np.float32)
    q0 = raw[(4096 + 2048) * 4:].view(np.uint32)
    dots = h[:4096].reshape(128, 32).astype(np.float64)
    t = h[4096:]
    Da, la, beta, m, E = (t[0:128], t[128:256], t[256:384], t[384:512], t[512:640])
    pos = t[640:768].view(np.uint32)
    mask = t[768:896].view(np.uint32)
    eta = t[1024:1056].astype(np.float64)
    Sq, Sv, na, nqt = t[1056], t[1057], int(t[1058]), int(t[1059])
    nr = t[1152:1280].astype(np.float64)
    sb = t[1280:1408].astype(np.float64)
    print(f"S={Sq} Sv={Sv} anchors={na} nqt={nqt}")
    perm = ix.export("PERM").astype(np.int64)
    rgrp = ix.export("RGRP")
    gstart = ix.export("GSTART")
    sizes = np.diff(gstart)
    print(f"anchor groups {len(sizes)}: rows per group median {np.median(sizes):.0f} mean {sizes.mean():.1f} max {sizes.max()}")
    Xh = X.cpu().numpy().astype(np.float64)
    Qh = Q.cpu().numpy().astype(np.float64)
    Xp = Xh[perm]
    qs = Qh[q0[:nqt]]
    delta = 2.0 ** -11
    worst, widths, npairs, bad = 0.0, [], 0, 0
    terms = {"E": [], "eta_n": [], "delta_d2": [], "d2": []}
    for i in range(128):
        if mask[i] == 0:
            continue
        p = int(pos[i])
        b = int(rgrp[p])
        blk = Xp[gstart[b]: gstart[b + 1]]
        anc = blk.mean(0).astype(np.float32).astype(np.float64)
        x = Xp[p]
        for j in range(nqt):
            if not (mask[i] >> j) & 1:
                continue
            K = ((qs[j] - anc) ** 2).sum()
            dt = K + beta[i] + m[i] * dots[i, j]
            err = E[i] + eta[j] * nr[i]
            lo, up = dt * (1 - delta) - err, dt * (1 + delta) + err
            ex = ((qs[j] - x) ** 2).sum()
            npairs += 1
            if not (lo <= ex <= up):
                bad += 1
                if bad < 10:
                    print(f"VIOLATION row {i} q {j}: exact {ex:.6g} lo {lo:.6g} up {up:.6g} d~ {dt:.6g}")
            widths.append((up - lo) / max(ex, 1e-30))
            terms["E"].append(E[i]); terms["eta_n"].append(eta[j] * nr[i]); terms["delta_d2"].append(delta * dt)
            terms["d2"].append(ex)
            worst = max(worst, abs(dt - ex) / max(ex, 1e-30))
    print(f"pairs {npairs}, violations {bad}, max |d~2 - d2|/d2 {worst:.3e}, "
          f"bound width/d2 median {np.median(widths) if widths else 0:.3e} max {max(widths) if widths else 0:.3e}")
    for kk, v in terms.items():
        if v:
            print(f"  {kk}: median {np.median(v):.3e} max {np.max(v):.3e}")
    print(f"  |s r| median {np.median(nr[mask != 0]):.3e} max {np.max(nr[mask != 0]):.3e}")
    sys.exit(1 if bad or npairs == 0 else 0)


if __name__ == "__main__":
    main()
