"""Where does the end-to-end rate lose against the device rate?  (experiment, c4)

Times K steps of the c4 query three ways, wall clock with a synchronize on both sides:
  device      ix.query on the device-resident batch (bench.py's `value` path)
  device+h2d  the same, plus an independent 154 MB pinned-host -> device copy per step on
              another stream (the copy competes for HBM/L2 but nothing waits on it)
  pipelined   blsh_query_pipelined over K pinned host batches (bench.py's `e2e` path)

    python tools/e2e_probe.py [--steps 10]
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
    ap.add_argument("--config", default="c4")
    ap.add_argument("--steps", type=int, default=10)
    a = ap.parse_args()
    cfg = synth.CONFIGS[a.config]
    X, Q = synth.make_dataset(cfg, backend="torch", device="cuda:0")
    ix = blsh.blsh_build(X, n_leaves=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index)
    kw = dict(probe=cfg.probe, n_probes=cfg.T, hierarchy=cfg.hierarchy)
    nq, k = Q.shape[0], cfg.k
    out = (torch.empty((nq, k), dtype=torch.int64, device="cuda"), torch.empty((nq, k), device="cuda"),
           torch.empty((nq,), dtype=torch.int64, device="cuda"))
    Qh = Q.cpu().pin_memory()
    Qd2 = torch.empty_like(Q)
    hout = (torch.empty((nq, k), dtype=torch.int64).pin_memory(), torch.empty((nq, k)).pin_memory(),
            torch.empty((nq,), dtype=torch.int64).pin_memory())
    side = torch.cuda.Stream()
    res = {}

    def run(name, fn):
        for _ in range(2):
            fn()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(a.steps):
            fn()
        torch.cuda.synchronize()
        ms = (time.perf_counter() - t0) * 1e3 / a.steps
        res[name] = {"ms_per_step": ms, "qps": nq / (ms * 1e-3)}
        print(name, json.dumps(res[name]), flush=True)

    run("device", lambda: ix.query(Q, k, out=out, **kw))

    def dev_h2d():
        with torch.cuda.stream(side):
            Qd2.copy_(Qh, non_blocking=True)
        ix.query(Q, k, out=out, **kw)
    run("device+h2d", dev_h2d)

    def piped():
        ix.query_pipelined([Qh] * a.steps, k, outs=[hout] * a.steps, **kw)
    for _ in range(1):
        piped()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    piped()
    torch.cuda.synchronize()
    ms = (time.perf_counter() - t0) * 1e3 / a.steps
    res["pipelined"] = {"ms_per_step": ms, "qps": nq / (ms * 1e-3)}
    print("pipelined", json.dumps(res["pipelined"]), flush=True)
    print(json.dumps(res))


if __name__ == "__main__":
    main()
