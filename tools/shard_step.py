"""Per-rank work of the leaf-sharded path, on ONE GPU.

    python tools/shard_step.py [--config c4] [--world 8]

Builds the full index and the shard of rank 0 of `world` (balanced contiguous leaf split
from the measured per-leaf loads, as bench.py's N > 1 runs do not yet; here the even split),
then times (CUDA events, 2 warm-ups, 5 timed calls) the single-GPU query and the shard's
query_packed on the same batch.  A shard routes the whole batch and runs a2-a5 only on its
own queries, so its step should approach 1/world of the single-GPU step.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
from paper_conf_icde_panm12_b200 import blsh  # noqa: E402


def timed(fn, reps=5):
    for _ in range(2):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c4")
    ap.add_argument("--world", type=int, default=8)
    a = ap.parse_args()
    cfg = synth.CONFIGS[a.config]
    X, Q = synth.make_dataset(cfg, backend="torch", device="cuda:0")
    kw = dict(probe=cfg.probe, n_probes=cfg.T)
    full = blsh.blsh_build(X, n_leaves=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index)
    ms_full = timed(lambda: full.query(Q, cfg.k, timing=True, **kw))
    st_full = full.stats()
    ids_f, d2_f, _ = full.query(Q, cfg.k, **kw)
    del full
    torch.cuda.empty_cache()
    out = dict(config=cfg.name, world=a.world, ms_single=ms_full, ms_shard={}, stage_single=dict(
        route_hash=st_full.ms_route_hash, probe=st_full.ms_probe, plan=st_full.ms_plan, shortlist=st_full.ms_shortlist))
    parts = []
    for r in range(a.world):
        sh = blsh.blsh_build(X, n_leaves=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index, rank=r, world=a.world)
        ms = timed(lambda: sh.query_packed(Q, cfg.k, timing=True, **kw), reps=3)
        out["ms_shard"][r] = ms
        st = sh.stats()
        out.setdefault("stage_shard", {})[r] = dict(nq_owned=st.n_active, route_hash=st.ms_route_hash,
                                                    probe=st.ms_probe, plan=st.ms_plan, screen=st.ms_screen,
                                                    rescore=st.ms_rescore, merge=st.ms_merge, total=st.ms_total,
                                                    items=st.n_items, launches=st.launches)
        parts.append(sh.query_packed(Q, cfg.k, **kw)[0].clone())
        del sh
        torch.cuda.empty_cache()
    mi, md = blsh.blsh_merge_topk(torch.cat(parts).contiguous(), a.world, Q.shape[0], cfg.k)
    torch.cuda.synchronize()
    out["merged_equals_single"] = bool(torch.equal(mi, ids_f) and torch.equal(md.view(torch.int32), d2_f.view(torch.int32)))
    out["max_shard_over_single"] = max(out["ms_shard"].values()) / ms_full
    print(json.dumps(out))


if __name__ == "__main__":
    main()
