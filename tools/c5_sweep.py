"""C5 recall / selectivity / throughput sweep (BASELINE configs[4]).

    python tools/c5_sweep.py [--out gpurun_out/c5_sweep.jsonl] [--config c5]

On n = 1M x 384 (synth c5), one B200, through the C ABI (blsh.py):
  * probes: T in {1, 2, 4, 8, 16, 32, 64} for three probe families -- Z^M multiprobe ([8]),
    the E8 lattice (DECODE + 240 roots, then the second ring for T > 241 is not reached
    here), and Morton-curve neighbours -- each at several bucket widths W = r10 * mult;
  * per point: recall@10 on the committed 1000-query oracle ground truth (bench_data/c5_gt.npz,
    tools/make_gt.py: oracle fp64 brute force, tie-aware as bench.py), selectivity (mean |A(q)| / n,
    P:45), queries/s over the full 100k batch (CUDA events, 1 warm-up + 3 timed calls), per-stage ms;
  * batch: B in {1, 10, 100, 1k, 10k, 100k} at each family's fastest point with recall >= 0.9 (else
    its best-recall point), with both short-list paths (the tiled TC screen and the warp short-list,
    BLSH_SHORTLIST=warp), queries/s and ms per batch.
One JSON object per line.  The leaf ceiling (fraction of the true 10-NN in the query's own leaf,
SURVEY D6) is printed once per W.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
from paper_conf_icde_panm12_b200 import blsh  # noqa: E402
import bench  # noqa: E402  (ground-truth loading, leaf ceiling, recall conventions)


FAMILIES = {
    "multiprobe": dict(quantizer=0, probe=1),
    "e8_lattice": dict(quantizer=1, probe=2),
    "morton_curve": dict(quantizer=0, probe=3),
}


def recall(g, X, Q, ids):
    """tie-aware recall@10 on the ground-truth sample (bench.recall_from_gt's rule, vectorised)."""
    qidx = torch.as_tensor(g["qidx"], device=Q.device)
    got = ids[qidx][:, :10]
    gi = torch.as_tensor(g["ids"][:, :10].astype(np.int64), device=Q.device)
    kth = torch.as_tensor(g["d2"][:, 9].astype(np.float64), device=Q.device)
    inset = (got[:, :, None] == gi[:, None, :]).any(-1)
    valid = got >= 0
    safe = torch.where(valid, got, torch.zeros_like(got))
    d = ((X[safe].double() - Q[qidx].double()[:, None, :]) ** 2).sum(-1)
    hit = valid & (inset | (d <= kth[:, None] * (1 + 1e-5)))
    return float(hit.float().mean())


def timed(ix, Q, k, kw, reps=3):
    ix.query(Q, k, **kw)
    torch.cuda.synchronize()
    s = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(reps):
        ix.query(Q, k, timing=True, **kw)
    e1.record(s)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps, ix.stats()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c5")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "c5_sweep.jsonl"))
    ap.add_argument("--probes", default="1,2,4,8,16,32,64")
    ap.add_argument("--wmult", default="2.83,4,5.66,8")
    ap.add_argument("--families", default="multiprobe,e8_lattice,morton_curve")
    ap.add_argument("--batches", default="1,10,100,1000,10000,100000")
    ap.add_argument("--points", default=None,
                    help="skip the probe sweep: batch sweep at family:W_mult:T[,...] (e.g. multiprobe:8:16)")
    a = ap.parse_args()
    cfg = synth.CONFIGS[a.config]
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    fo = open(a.out, "w")

    def emit(row):
        print(json.dumps(row), flush=True)
        fo.write(json.dumps(row) + "\n")
        fo.flush()

    X, Q = synth.make_dataset(cfg, backend="torch", device="cuda:0")
    torch.cuda.synchronize()
    g = bench._gt_file(cfg, X, Q)
    if g is None:
        raise SystemExit(f"no matching bench_data/{cfg.name}_gt.npz (tools/make_gt.py --config {cfg.name} --sample 1000)")
    r10 = float(np.median(np.sqrt(g["d2"][:, 9])))
    emit(dict(kind="dataset", config=cfg.name, n=cfg.n, d=cfg.d, nq=Q.shape[0], G=cfg.G, M=cfg.M, k=cfg.k,
              r10=r10, gt="bench_data/%s_gt.npz (%d queries, oracle fp64 brute force)" % (cfg.name, len(g["qidx"]))))
    k = cfg.k
    best = {}
    if a.points:
        for pt in a.points.split(","):
            fam, wm, T = pt.split(":")
            best[fam] = (None, dict(W=float(wm) * r10, T=int(T), recall10=None))
    for fam in ([] if a.points else a.families.split(",")):
        fk = FAMILIES[fam]
        for wm in [float(w) for w in a.wmult.split(",")]:
            W = wm * r10
            t0 = time.time()
            ix = blsh.blsh_build(X, n_leaves=cfg.G, M=cfg.M, W=W, seed=cfg.seed_index, quantizer=fk["quantizer"])
            torch.cuda.synchronize()
            bt = time.time() - t0
            ceiling = None
            for T in [int(t) for t in a.probes.split(",")]:
                probe = fk["probe"] if T > 1 else 0
                kw = dict(probe=probe, n_probes=T)
                ids, d2, nc = ix.query(Q, k, keep_stages=True, **kw)
                if ceiling is None:
                    ceiling = bench.leaf_ceiling(cfg, ix, X, Q)
                rec = recall(g, X, Q, ids)
                ms, st = timed(ix, Q, k, kw)
                row = dict(kind="probe", family=fam, W_mult=wm, W=W, T=T, recall10=rec, leaf_ceiling=ceiling,
                           selectivity=float(nc.double().mean()) / cfg.n, mean_cand=float(nc.double().mean()),
                           qps=Q.shape[0] / (ms * 1e-3), ms=ms, build_s=bt,
                           shortlist={0: "warp", 1: "simt_tiled", 2: "tc_screen"}[st.tiled],
                           ms_route_hash=st.ms_route_hash, ms_probe=st.ms_probe, ms_plan=st.ms_plan,
                           ms_screen=st.ms_screen, ms_rescore=st.ms_rescore, ms_shortlist=st.ms_shortlist)
                emit(row)
                key = fam
                ok = row["recall10"] >= 0.9
                cur = best.get(key)
                if cur is None or (ok and (not cur[0] or row["qps"] > cur[1]["qps"])) or \
                        (not ok and not cur[0] and row["recall10"] > cur[1]["recall10"]):
                    best[key] = (ok, row)
            ix.close()
    # batch sweep at each family's operating point, both short-list paths
    for fam, (ok, row) in best.items():
        fk = FAMILIES[fam]
        ix = blsh.blsh_build(X, n_leaves=cfg.G, M=cfg.M, W=row["W"], seed=cfg.seed_index, quantizer=fk["quantizer"])
        kw = dict(probe=fk["probe"] if row["T"] > 1 else 0, n_probes=row["T"])
        for B in [int(b) for b in a.batches.split(",")]:
            Qb = Q[:B].contiguous()
            for path in ("tc", "warp"):
                if path == "warp":
                    os.environ["BLSH_SHORTLIST"] = "warp"
                else:
                    os.environ.pop("BLSH_SHORTLIST", None)
                reps = max(3, min(200, 200000 // max(B, 1)))
                ms, st = timed(ix, Qb, k, kw, reps=reps)
                emit(dict(kind="batch", family=fam, at_recall_gate=ok, W=row["W"], T=row["T"],
                          recall10_full_batch=row["recall10"], batch=B, path=path,
                          shortlist={0: "warp", 1: "simt_tiled", 2: "tc_screen"}[st.tiled],
                          qps=B / (ms * 1e-3), ms_per_batch=ms, ms_shortlist=st.ms_shortlist,
                          ms_screen=st.ms_screen, mean_cand=st.total_cand / max(B, 1),
                          shortlist_bytes=st.shortlist_bytes,
                          shortlist_gbs=st.shortlist_bytes / (st.ms_shortlist * 1e-3) / 1e9 if st.ms_shortlist > 0 else None))
        os.environ.pop("BLSH_SHORTLIST", None)
        ix.close()
    fo.close()


if __name__ == "__main__":
    main()
