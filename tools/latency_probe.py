"""Small-batch latency breakdown (experiment): per batch size, the wall time of one
blsh_query call (host work + GPU), the GPU span of the call (CUDA events inside the
library, stats.ms_total) and the per-stage GPU times.

    python tools/latency_probe.py [--config c5] [--batches 1,10,100]
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icde_panm12_b200 import blsh  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c5")
    ap.add_argument("--batches", default="1,10,100,1000")
    ap.add_argument("--reps", type=int, default=200)
    a = ap.parse_args()
    cfg = synth.CONFIGS[a.config]
    X, Q = synth.make_dataset(cfg, backend="torch", device="cuda:0")
    ix = blsh.blsh_build(X, n_leaves=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index)
    kw = dict(probe=cfg.probe, n_probes=cfg.T, hierarchy=cfg.hierarchy)
    for B in [int(b) for b in a.batches.split(",")]:
        Qb = Q[:B].contiguous()
        out = (torch.empty((B, cfg.k), dtype=torch.int64, device="cuda"), torch.empty((B, cfg.k), device="cuda"),
               torch.empty((B,), dtype=torch.int64, device="cuda"))
        for _ in range(10):
            ix.query(Qb, cfg.k, out=out, **kw)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(a.reps):
            ix.query(Qb, cfg.k, out=out, **kw)
        torch.cuda.synchronize()
        wall = (time.perf_counter() - t0) * 1e3 / a.reps
        ix.query(Qb, cfg.k, out=out, timing=True, **kw)
        st = ix.stats()
        row = dict(batch=B, wall_ms=wall, gpu_span_ms=st.ms_total, route_hash=st.ms_route_hash, probe=st.ms_probe,
                   plan=st.ms_plan, shortlist=st.ms_shortlist, merge=st.ms_merge, launches=st.launches,
                   path={0: "warp", 1: "simt_tiled", 2: "tc_screen"}[st.tiled])
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
