"""Drive every kernel family once on c1-sized inputs (for compute-sanitizer).

    compute-sanitizer --tool {memcheck,racecheck,synccheck,initcheck} python tools/sanitize_c1.py

Build (Z^M and E8, L = 2, per-leaf W), then queries that reach the route/hash,
probe (standard, multiprobe, E8 lattice + recursive ring, Morton curve),
hierarchy (Morton prefixes, E8 code hierarchy), the tiled tensor-core
short-list + exact rescoring, the SIMT tiled short-list (k = 50), the warp
short-list, large-k selection and the multi-table union.  Prints one line per
case; the sanitizer's own report is the result.
"""
from __future__ import annotations

import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icde_panm12_b200 import blsh  # noqa: E402


def main():
    # 1 200 queries: batches above 1 024 take the query-tiled paths
    X, Q = synth.make_dataset(synth.CONFIGS["c1"], nq=1200)
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    cases = [
        (dict(), dict(probe=0, n_probes=1), 10),
        (dict(), dict(probe=1, n_probes=16), 10),        # TC screen (k <= 32)
        (dict(), dict(probe=1, n_probes=16), 50),        # fp16 screen, KT = 64
        (dict(), dict(probe=1, n_probes=8), 200),        # large k on the fp16 screen (k_tc_emit + select)
        (dict(), dict(probe=1, n_probes=8), 600),        # k > 512: warp short-list emit + select
        (dict(), dict(probe=1, n_probes=8, hierarchy=1), 10),
        (dict(), dict(probe=3, n_probes=6), 10),
        (dict(quantizer=1), dict(probe=2, n_probes=250), 10),
        (dict(quantizer=1), dict(probe=2, n_probes=256, min_cand=200), 10),   # R33 recursion
        (dict(quantizer=1), dict(probe=2, n_probes=8, hierarchy=1), 10),
        (dict(n_tables=2), dict(probe=1, n_probes=4), 10),
        (dict(W_rule=1), dict(probe=1, n_probes=4), 10),
    ]
    for bk, qk, k in cases:
        ix = blsh.blsh_build(Xd, n_leaves=4, M=8, W=4.0, seed=42, **bk)
        ids, d2, nc = ix.query(Qd, k, **qk)
        torch.cuda.synchronize()
        st = ix.stats()
        print(f"build {bk} query {qk} k={k}: tiled={st.tiled} mean|A|={float(nc.double().mean()):.1f}", flush=True)
        ix.close()
    # small batch (sync-free warp path), the pipelined host-batch API
    ix = blsh.blsh_build(Xd, n_leaves=4, M=8, W=4.0, seed=42)
    ix.query(Qd[:3], 10, probe=1, n_probes=16)
    ix.query(Qd[:100], 60, probe=1, n_probes=16, hierarchy=1)
    Qh = Q[:200].copy()
    ix.query_pipelined([Qh, Qh, Qh], 10, probe=1, n_probes=8)
    torch.cuda.synchronize()
    print("small batches + pipelined ok", flush=True)
    # forced warp short-list and SIMT tiled
    for mode in ("warp", "simt"):
        os.environ["BLSH_SHORTLIST"] = mode
        ix.query(Qd, 10, probe=1, n_probes=16)
        torch.cuda.synchronize()
        print(f"{mode} short-list ok", flush=True)
    os.environ.pop("BLSH_SHORTLIST", None)
    ix.close()


if __name__ == "__main__":
    main()
