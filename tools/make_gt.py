"""Write the oracle's exact k-NN ground truth for a bench workload sample.

    python tools/make_gt.py --config c4 [--sample 200]

Generates the workload exactly as bench.py does (synth/, torch backend on
cuda:0), draws a fixed sample of query indices, and runs the ORACLE's fp64
brute force (oracle.bruteforce) on the host.  Stores
bench_data/<config>_gt.npz = {n, nq, qidx, ids, d2, fp_x, fp_q}; the
fingerprints let bench.py refuse a file that does not match its data.
No value in the file comes from the CUDA path.
"""
from __future__ import annotations

import argparse
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c4")
    ap.add_argument("--sample", type=int, default=200)
    ap.add_argument("--k", type=int, default=50)
    ap.add_argument("--out-dir", default=os.path.join(ROOT, "bench_data"))
    a = ap.parse_args()
    import torch
    cfg = synth.CONFIGS[a.config]
    X, Q = synth.make_dataset(cfg, backend="torch", device="cuda:0")
    rng = np.random.default_rng(12345)
    qidx = np.sort(rng.choice(Q.shape[0], min(a.sample, Q.shape[0]), replace=False))
    fp_x = float(X[:: max(1, X.shape[0] // 997)].double().sum())
    fp_q = float(Q[torch.as_tensor(qidx, device=Q.device)].double().sum())
    Xh = X.cpu().numpy()
    Qs = Q.cpu().numpy()[qidx]
    del X, Q
    t0 = time.time()
    ids, d2 = oracle.bruteforce(Xh, Qs, a.k)
    print(f"brute force {len(qidx)} x {Xh.shape[0]} in {time.time() - t0:.1f}s on {oracle.num_threads()} threads")
    os.makedirs(a.out_dir, exist_ok=True)
    out = os.path.join(a.out_dir, f"{cfg.name}_gt.npz")
    np.savez_compressed(out, n=Xh.shape[0], nq=cfg.nq, qidx=qidx, ids=ids, d2=d2, fp_x=fp_x, fp_q=fp_q)
    print("wrote", out)


if __name__ == "__main__":
    main()
