"""Summarise a C5 sweep (tools/c5_sweep.py output) as markdown tables: per probe family and W,
recall@10 / selectivity / queries/s for every T; the batch surface at each family's point.

    python tools/c5_table.py profiles/r02/c5_sweep_final.jsonl
"""
from __future__ import annotations

import collections
import json
import sys


def main(path):
    rows = [json.loads(l) for l in open(path)]
    probe = [r for r in rows if r.get("kind") == "probe"]
    batch = [r for r in rows if r.get("kind") == "batch"]
    by = collections.defaultdict(list)
    for r in probe:
        by[(r["family"], r["W_mult"])].append(r)
    Ts = sorted({r["T"] for r in probe})
    print("| family | W / r10 | " + " | ".join(f"T = {t}" for t in Ts) + " |")
    print("|---|---|" + "---|" * len(Ts))
    for (fam, wm), rs in sorted(by.items()):
        cell = {r["T"]: r for r in rs}
        out = []
        for t in Ts:
            r = cell.get(t)
            out.append("" if r is None else f"{r['recall10']:.3f} / {100 * r['selectivity']:.3f}% / {r['qps'] / 1e6:.1f} M")
        print(f"| {fam} | {wm:g} | " + " | ".join(out) + " |")
    print()
    print("(cells: recall@10 / selectivity / queries/s of the full 100k batch)")
    print()
    bb = collections.defaultdict(dict)
    for r in batch:
        bb[(r["family"], r["path"])][r["batch"]] = r
    Bs = sorted({r["batch"] for r in batch})
    print("| family, short-list path | " + " | ".join(f"batch {b}" for b in Bs) + " |")
    print("|---|" + "---|" * len(Bs))
    for (fam, path), d in sorted(bb.items()):
        print(f"| {fam}, {path} | " + " | ".join(
            f"{d[b]['qps'] / 1e3:.1f} k ({d[b]['ms_per_batch']:.2f} ms)" if b in d else "" for b in Bs) + " |")


if __name__ == "__main__":
    main(sys.argv[1])
