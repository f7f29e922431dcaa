"""Helpers for GPU-vs-oracle parity tests (test infrastructure)."""
from __future__ import annotations

import numpy as np

TOL = 1e-5   # north star: distances within 1e-5 relative


def gpu_candidates(ix, T: int):
    """Candidate id sets A(q) of the last GPU query (keep_stages=True), via
    the exported intervals and table permutation."""
    iv = ix.export("Q_INTERVALS").reshape(-1, T + 1, 2)
    perm = ix.export("PERM")
    out = []
    for q in range(iv.shape[0]):
        parts = [perm[s:e] for s, e in iv[q] if e > s]
        ids = np.concatenate(parts) if parts else np.zeros(0, np.int64)
        out.append(np.sort(ids))
    return out


def exact_d2(X, Q, q, ids):
    ids = np.asarray(ids)
    return ((X[ids].astype(np.float64) - Q[q].astype(np.float64)) ** 2).sum(1)


def check_topk(ids_g, d2_g, ids_o, d2_o, X, Q, cands=None, tol=TOL):
    """(i) position-wise distances within tol of the oracle's;
    (ii) every GPU id is a candidate and its exact distance matches the
    reported one; (iii) id sets differ only at ties within tol of the k-th."""
    nq, k = ids_o.shape
    for q in range(nq):
        vo = np.isfinite(d2_o[q])
        vg = np.isfinite(d2_g[q])
        assert np.array_equal(vo, vg), f"q={q}: padding differs"
        assert np.all(ids_g[q][~vg] == -1)
        m = int(vo.sum())
        if m == 0:
            continue
        do, dg = d2_o[q, :m].astype(np.float64), d2_g[q, :m].astype(np.float64)
        assert np.all(np.abs(dg - do) <= tol * np.maximum(do, 1e-30) + 1e-30), f"q={q}: distances differ"
        gi = ids_g[q, :m]
        assert len(set(gi.tolist())) == m, f"q={q}: duplicate ids"
        if cands is not None:
            cs = set(cands[q].tolist())
            assert all(int(i) in cs for i in gi), f"q={q}: id outside A(q)"
        ex = exact_d2(X, Q, q, gi)
        assert np.all(np.abs(ex - dg) <= tol * np.maximum(ex, 1e-30) + 1e-30), f"q={q}: reported d2 wrong"
        kth = do[-1]
        diff = set(gi.tolist()) ^ set(ids_o[q, :m].tolist())
        for i in diff:
            e = exact_d2(X, Q, q, [i])[0]
            assert abs(e - kth) <= tol * max(kth, 1e-30) + 1e-30, f"q={q}: id {i} differs beyond a tie"


def key_rows(a):
    """[n,2] uint64 (hi, lo) -> list of python ints."""
    return [(int(h) << 64) | int(l) for h, l in a]
