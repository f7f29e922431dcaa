#!/usr/bin/env python
"""bench.py -- Bi-level LSH query hot path on B200 (BASELINE.json metric).

A *step* is one pass of the whole query hot path (route + hash, probe
generation + lookup, short-list, top-k merge; + NCCL all-gather and merge when
N > 1) over one batch of synthetic queries against a resident index.  The
index build (b1-b4) happens before the timed region and is reported as
``build_s``.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c4] [--impl ours|reference]

N > 1 runs under torchrun (one process per GPU, NCCL): every rank builds the
shard of RP-tree leaves it owns, routes the whole batch, answers the queries
of its leaves, then the per-rank packed top-k lists are all-gathered and
merged.  Rank 0 prints one JSON line.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "queries/sec at recall@10>=0.9 (1/2/4/8 B200); short-list HBM GB/s vs peak"
UNIT = "queries/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="c4")
    ap.add_argument("--W", type=float, default=None)
    ap.add_argument("--T", type=int, default=None)
    ap.add_argument("--nq", type=int, default=None)
    ap.add_argument("--n", type=int, default=None)
    ap.add_argument("--k", type=int, default=None)
    ap.add_argument("--L", type=int, default=None, help="hash tables per leaf (P:43)")
    ap.add_argument("--G", type=int, default=None)
    ap.add_argument("--probe", type=int, default=None, help="0 standard, 1 multiprobe, 2 E8 lattice")
    ap.add_argument("--quantizer", type=int, default=None, help="0 Z^M, 1 E8")
    ap.add_argument("--hierarchy", type=int, default=None)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--cpu-sample-s", type=float, default=15.0, help="target seconds of oracle query work")
    ap.add_argument("--nvtx", action="store_true", help="NVTX range around the timed region (ncu filtering)")
    return ap.parse_args()


def load_cfg(a):
    import synth
    from dataclasses import replace
    cfg = synth.CONFIGS[a.config]
    kw = {}
    if a.W is not None:
        kw["W"] = a.W
    if a.T is not None:
        kw["T"] = a.T
        kw["probe"] = 1 if a.T > 1 else 0
    if a.nq is not None:
        kw["nq"] = a.nq
    if a.n is not None:
        kw["n"] = a.n
    for f in ("k", "L", "G", "probe", "quantizer", "hierarchy"):
        if getattr(a, f) is not None:
            kw[f] = getattr(a, f)
    return replace(cfg, **kw) if kw else cfg


def workload_str(cfg):
    probe = {0: "standard", 1: f"multiprobe T={cfg.T}", 2: f"E8 lattice T={cfg.T}",
             3: f"Morton-curve neighbours T={cfg.T}"}[cfg.probe]
    hier = " + Morton hierarchy (tau=median)" if cfg.hierarchy else ""
    if cfg.L > 1:
        hier += f", L={cfg.L} tables"
    return (f"{cfg.name}: n={cfg.n} d={cfg.d} Gaussian-mixture (C={cfg.n_clusters}, spread={cfg.spread}), "
            f"{cfg.nq} queries, k={cfg.k}, RP-tree G={cfg.G}, M={cfg.M}, W={cfg.W:g}, {probe}{hier}")


# --- clocks -------------------------------------------------------------------------

class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")
    NAMES = ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap")

    def __init__(self, gpu_id: str):
        self.gpu_id = gpu_id
        self.lines = []
        self.proc = None
        self.thread = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", self.gpu_id, f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
            return
        self.thread = threading.Thread(target=self._read, daemon=True)
        self.thread.start()

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        if self.thread:
            self.thread.join(timeout=5)
        sm, mx, reasons = [], [], set()
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for name, v in zip(self.NAMES, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(name)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm)}


def gpu_smi_id(torch, dev):
    p = torch.cuda.get_device_properties(dev)
    try:
        return f"{p.pci_domain_id:08X}:{p.pci_bus_id:02X}:{p.pci_device_id:02X}.0"
    except AttributeError:
        return str(dev)


# --- helpers --------------------------------------------------------------------------

def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            m = json.load(f)
        return float(m["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def source_sha() -> str:
    """sha256 (16 hex) of the library's CUDA/C++ sources: ties an ncu capture to the build it measured."""
    import glob
    import hashlib
    h = hashlib.sha256()
    for f in sorted(glob.glob(os.path.join(ROOT, "paper_conf_icde_panm12_b200", "csrc", "*"))):
        with open(f, "rb") as fh:
            h.update(os.path.basename(f).encode())
            h.update(fh.read())
    return h.hexdigest()[:16]


def traffic_for(workload: str, kernel: str):
    """(dram read+write bytes per launch, entry) from a committed ncu --set full capture of this
    kernel and workload, ONLY if the capture was taken on the current sources (source_sha);
    otherwise (None, reason)."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            entries = json.load(f)
    except Exception:
        return None, "no profiles/traffic.json"
    cur = source_sha()
    hit, stale = None, None
    for t in entries if isinstance(entries, list) else [entries]:
        if t.get("workload") == workload and t.get("kernel", "").split("<")[0] == kernel:
            if t.get("source_sha") == cur:
                hit = t
            else:
                stale = t
    if hit:
        return hit.get("bytes_per_launch"), hit
    if stale:
        return None, f"latest ncu capture of {kernel} is of another build ({stale.get('source_sha', 'untagged')})"
    return None, f"no ncu capture of {kernel} on this workload"


def distinct_candidate_rows(ix, T: int, n_owned: int) -> int:
    """Table rows that are candidates of at least one query of the last (keep_stages) query:
    the union of every query's intervals, by a difference array (torch, measurement only)."""
    import torch
    iv = torch.as_tensor(ix.export("Q_INTERVALS").reshape(-1, 2).astype(np.int64), device="cuda")
    iv = iv[iv[:, 1] > iv[:, 0]]
    diff = torch.zeros(n_owned + 1, dtype=torch.int32, device="cuda")
    ones = torch.ones(iv.shape[0], dtype=torch.int32, device="cuda")
    diff.index_add_(0, iv[:, 0], ones)
    diff.index_add_(0, iv[:, 1], -ones)
    return int((torch.cumsum(diff[:-1], 0) > 0).sum().item())


def l2_copy_gbs() -> float:
    """L2-resident copy bandwidth (read + write bytes / time) of a 24 MB torch copy, best of 50:
    the denominator for short-lists whose table fits in the 126 MB L2."""
    import torch
    a = torch.empty(6 * 1024 * 1024, dtype=torch.float32, device="cuda")
    b = torch.empty_like(a)
    for _ in range(5):
        b.copy_(a)
    best = None
    for _ in range(50):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(20):
            b.copy_(a)
        e1.record()
        torch.cuda.synchronize()
        t = e0.elapsed_time(e1) / 20
        best = t if best is None else min(best, t)
    return 2 * a.numel() * 4 / (best * 1e-3) / 1e9


def leaf_ceiling(cfg, ix, X, Q):
    """SURVEY D6 leaf ceiling: the fraction of the ground-truth 10-NN (committed oracle sample) that
    lie in the query's own RP-tree leaf -- the recall@10 no probing of that leaf can exceed.
    Point leaves from the table directory (PERM, UOFF, LEAF_U), query leaves from the last
    keep_stages query (Q_LEAF).  None without a matching ground-truth file."""
    g = _gt_file(cfg, X, Q)
    if g is None:
        return None
    perm = ix.export("PERM").astype(np.int64)
    uoff = ix.export("UOFF").astype(np.int64)
    leaf_u = ix.export("LEAF_U").astype(np.int64)
    row_start = uoff[leaf_u]                               # first table row of every leaf (+ end)
    pos_leaf = np.searchsorted(row_start, np.arange(perm.shape[0]), side="right") - 1
    pt_leaf = np.full(X.shape[0], -1, np.int64)
    pt_leaf[perm] = pos_leaf
    qleaf = ix.export("Q_LEAF").astype(np.int64)[g["qidx"]]
    gi = g["ids"][:, :10]
    return float((pt_leaf[gi] == qleaf[:, None]).mean())


def _gt_file(cfg, X, Q):
    """The committed ground-truth sample of this workload if its size and fingerprints match."""
    path = os.path.join(ROOT, "bench_data", f"{cfg.name}_gt.npz")
    if not os.path.exists(path):
        return None
    g = np.load(path)
    if int(g["n"]) != X.shape[0] or int(g["nq"]) != Q.shape[0]:
        return None
    import torch
    qidx = torch.as_tensor(g["qidx"], device=Q.device)
    fpx = float(X[:: max(1, X.shape[0] // 997)].double().sum())
    fpq = float(Q[qidx].double().sum())
    if abs(fpx - float(g["fp_x"])) > 1e-6 * max(1.0, abs(float(g["fp_x"]))) or \
       abs(fpq - float(g["fp_q"])) > 1e-6 * max(1.0, abs(float(g["fp_q"]))):
        return None
    return g


def error_ratio(gt_d2, our_d2):
    """Eq. 4: kappa = (1/k) sum_i |v - N(v)_i| / |v - I(v)_i| over the sample
    (0/0 = 1; a padded answer contributes 0), from fp64 ground-truth and reported d^2."""
    g = np.sqrt(np.maximum(np.asarray(gt_d2, np.float64), 0.0))
    o = np.sqrt(np.maximum(np.asarray(our_d2, np.float64), 0.0))
    with np.errstate(divide="ignore", invalid="ignore"):
        r = np.where(o > 0, g / o, np.where(g == 0, 1.0, 0.0))
    r[~np.isfinite(o)] = 0.0
    return float(r.mean())


def recall_from_gt(cfg, X, Q, ids_dev, d2_dev=None):
    """recall@10 on the committed oracle ground-truth sample (tools/make_gt.py), tie-aware (C9);
    with d2_dev, also the error ratio of Eq. 4 on the same sample (stored as self.kappa)."""
    import torch
    recall_from_gt.kappa = None
    path = os.path.join(ROOT, "bench_data", f"{cfg.name}_gt.npz")
    if not os.path.exists(path) and X.shape[0] <= 2_000_000 and ids_dev.shape[1] >= 10:
        # no committed ground truth: exact 10-NN of a fixed 200-query sample by the oracle's fp64 brute force
        import oracle
        qidx = np.arange(0, Q.shape[0], max(1, Q.shape[0] // 200))[:200]
        gi, gd = oracle.bruteforce(X.cpu().numpy(), Q[torch.as_tensor(qidx, device=Q.device)].cpu().numpy(), 10)
        got = ids_dev[torch.as_tensor(qidx, device=ids_dev.device)][:, :10].cpu().numpy()
        if d2_dev is not None:
            recall_from_gt.kappa = error_ratio(gd, d2_dev[torch.as_tensor(qidx, device=d2_dev.device)][:, :10].cpu().numpy())
        hits = 0
        for r in range(len(qidx)):
            gs = set(gi[r].tolist())
            for i in got[r]:
                if i >= 0 and (int(i) in gs or float(((X[int(i)].double() - Q[int(qidx[r])].double()) ** 2).sum())
                               <= float(gd[r, 9]) * (1 + 1e-5)):
                    hits += 1
        return hits / (10.0 * len(qidx)), f"{len(qidx)} queries, oracle fp64 brute force (computed in this run)"
    if not os.path.exists(path):
        return None, "no ground-truth file"
    g = np.load(path)
    if int(g["n"]) != X.shape[0] or int(g["nq"]) != Q.shape[0]:
        return None, "ground truth for another size"
    qidx = torch.as_tensor(g["qidx"], device=Q.device)
    fpx = float(X[:: max(1, X.shape[0] // 997)].double().sum())
    fpq = float(Q[qidx].double().sum())
    if abs(fpx - float(g["fp_x"])) > 1e-6 * max(1.0, abs(float(g["fp_x"]))) or \
       abs(fpq - float(g["fp_q"])) > 1e-6 * max(1.0, abs(float(g["fp_q"]))):
        return None, "ground-truth fingerprint mismatch"
    gi, gd = g["ids"][:, :10], g["d2"][:, :10].astype(np.float64)
    got = ids_dev[qidx][:, :10].cpu().numpy()
    if d2_dev is not None:
        recall_from_gt.kappa = error_ratio(gd, d2_dev[qidx][:, :10].cpu().numpy())
    Xs = X
    hits = 0
    for r in range(len(gi)):
        kth = gd[r, 9]
        gs = set(gi[r].tolist())
        for i in got[r]:
            if i < 0:
                continue
            if int(i) in gs:
                hits += 1
            else:
                e = float(((Xs[int(i)].double() - Q[int(g["qidx"][r])].double()) ** 2).sum())
                if e <= kth * (1 + 1e-5):
                    hits += 1
    return hits / (10.0 * len(gi)), f"{len(gi)} queries, oracle fp64 brute force"


# --- our arm ------------------------------------------------------------------------

def run_ours(a):
    import torch
    import torch.distributed as dist
    import synth
    from paper_conf_icde_panm12_b200 import blsh
    from paper_conf_icde_panm12_b200.sharded import ShardedIndex

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    cfg = load_cfg(a)
    t0 = time.time()
    X, Q = synth.make_dataset(cfg, backend="torch", device=f"cuda:{local}")
    torch.cuda.synchronize()
    gen_s = time.time() - t0
    t0 = time.time()
    ix = blsh.blsh_build(X, n_leaves=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index, quantizer=cfg.quantizer,
                         rank=rank, world=world, n_tables=cfg.L)
    sh = ShardedIndex(ix) if world > 1 else None
    torch.cuda.synchronize()
    build_s = time.time() - t0
    info = ix.info()
    nq, k = Q.shape[0], cfg.k
    kw = dict(probe=cfg.probe, n_probes=cfg.T, hierarchy=cfg.hierarchy, min_cand=cfg.min_cand)
    out_ids = torch.empty((nq, k), dtype=torch.int64, device=dev)
    out_d2 = torch.empty((nq, k), dtype=torch.float32, device=dev)
    out_nc = torch.empty((nq,), dtype=torch.int64, device=dev)
    pk = torch.empty((nq, k), dtype=torch.int64, device=dev)
    stats = []

    def step(timing):
        if world == 1:
            ix.query(Q, k, timing=timing, out=(out_ids, out_d2, out_nc), **kw)
            stats.append(ix.stats())
            return 0
        # leaf-sharded: this rank's packed lists -> NCCL all-gather -> blsh_merge_topk (sharded.py)
        sh.query(Q, k, timing=timing, out=(out_ids, out_d2), packed_out=(pk, out_nc), **kw)
        stats.append(ix.stats())
        return 1 + (1 if cfg.hierarchy and not cfg.min_cand else 0)

    for _ in range(a.warmup):
        step(False)
    stats.clear()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = ClockSampler(gpu_smi_id(torch, dev)) if rank == 0 else None
    if clk:
        clk.start()
        time.sleep(0.3)
    stream = torch.cuda.current_stream(dev)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if a.nvtx:
        torch.cuda.nvtx.range_push("timed")
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    e0.record(stream)
    extra = 0
    for _ in range(a.steps):
        extra += step(True)
    e1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    if a.nvtx:
        torch.cuda.nvtx.range_pop()
    ms = e0.elapsed_time(e1)
    t_ms = torch.tensor([ms], device=dev, dtype=torch.float64)
    if world > 1:
        dist.all_reduce(t_ms, op=dist.ReduceOp.MAX)
    ms = float(t_ms.item())
    clocks = clk.stop() if clk else None
    sl_ms = sum(s.ms_shortlist for s in stats) / max(len(stats), 1)
    sl_bytes = sum(s.shortlist_bytes for s in stats) / max(len(stats), 1)
    total_cand = sum(s.total_cand for s in stats) / max(len(stats), 1)
    launches = sum(s.launches for s in stats) + extra
    recall, recall_note = (None, "sharded") if world > 1 and rank != 0 else recall_from_gt(cfg, X, Q, out_ids, out_d2)
    kappa = getattr(recall_from_gt, "kappa", None)
    shard_load = None
    if world > 1:   # query skew across leaves -> per-rank load of the last step
        ld = sh.load_stats()
        cands = [c for _, c in ld]
        shard_load = {"queries": [q for q, _ in ld], "candidates": cands,
                      "imbalance": max(cands) / max(1e-9, sum(cands) / len(cands))}

    # end to end through the C ABI with host buffers (pinned), copies inside the timed region
    e2e = None
    if not a.no_e2e:
        Qh = Q.cpu().pin_memory()
        hi = torch.empty((nq, k), dtype=torch.int64).pin_memory()
        hd = torch.empty((nq, k), dtype=torch.float32).pin_memory()
        hn = torch.empty((nq,), dtype=torch.int64).pin_memory()
        hpk = torch.empty((nq, k), dtype=torch.int64, device=dev)

        def e2e_steps(n):
            if world == 1:
                # the serving call: n host batches through blsh_query_pipelined (batch b + 1's upload and
                # batch b - 1's download overlap batch b's search; every copy inside the timed region)
                ix.query_pipelined([Qh] * n, k, outs=[(hi, hd, hn)] * n, **kw)
            else:
                for _ in range(n):
                    sh.query(Qh, k, out=(hi, hd), packed_out=(hpk, out_nc), **kw)

        e2e_steps(max(1, a.warmup // 2))
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        t1 = time.perf_counter()
        e2e_steps(a.steps)
        torch.cuda.synchronize()
        te = torch.tensor([time.perf_counter() - t1], device=dev, dtype=torch.float64)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        h2d = nq * cfg.d * 4
        d2h = nq * k * 12 + (nq * 8 if world == 1 else 0)
        e2e = {"value": nq * a.steps / float(te.item()), "unit": UNIT, "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": d2h,
               "api": "blsh_query_pipelined (pinned host batches, copies overlapped)" if world == 1
               else "blsh_query_packed + NCCL all-gather + blsh_merge_topk (pinned host batch, host answers)"}

    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        cpu = cpu_baseline(cfg, X, Q, a.cpu_sample_s)

    if rank == 0:
        peak, peak_src = peaks()
        wl = workload_str(cfg)
        kind = stats[0].tiled if stats else 0
        avg = lambda f: sum(getattr(s, f) for s in stats) / max(len(stats), 1)
        skind = stats[0].screen_kind if stats else 0
        kname = {0: "k_shortlist", 1: "k_shortlist_tiled", 2: "k_shortlist_tc"}[kind]
        if kind == 2 and skind == 1:
            kname = "k_screen_f16"
        if kind:
            k_ms = avg("ms_screen")
            union_bytes = avg("union_bytes")
            row_bytes = stats[0].screen_row_bytes
        else:
            k_ms = sl_ms
            union_bytes = sl_bytes
            row_bytes = 4 * cfg.d + 4
        # Algorithmic bytes of one launch (SURVEY §8(d) D4 with reuse): every table row that is a
        # candidate of some query of the batch has to reach the SMs at least once, at the width the
        # kernel reads it (fp16 screen: 2 dr + 16 B; fp32 kernels: 4 d_stride (+ metadata)); plus
        # the query batch once.  Bytes served again from L2 (tiles sharing rows) are NOT counted.
        distinct = None
        ceiling = None
        if world == 1:
            ix.query(Q, k, keep_stages=True, **kw)
            if cfg.L == 1:
                distinct = distinct_candidate_rows(ix, cfg.T, info.n_owned)
            ceiling = leaf_ceiling(cfg, ix, X, Q)
        if distinct is None:
            distinct = min(total_cand, info.n_owned)
        per_row = (row_bytes - 16) if (kind == 2 and skind == 1) else row_bytes   # rowinfo is per union row, not per table row
        alg_bytes = distinct * per_row + nq * 4 * info.d_stride
        achieved = alg_bytes / (k_ms * 1e-3) / 1e9 if k_ms > 0 else None
        traffic, tnote = traffic_for(wl, kname)
        l2_resident = info.n_owned * per_row <= 96e6
        l2_peak = l2_copy_gbs() if l2_resident else None
        bound, pk = ("l2", l2_peak) if l2_resident else ("hbm", peak)
        roof = {"kernel": kname, "bound": bound, "achieved": achieved, "peak": pk, "unit": "GB/s",
                "frac": (achieved / pk) if achieved else None, "traffic": traffic,
                "peak_source": ("measured in this run: L2-resident 24 MB torch copy" if l2_resident else peak_src),
                "algorithmic_bytes_per_launch": alg_bytes,
                "algorithmic_note": f"{distinct} distinct candidate rows x {per_row} B + the query batch",
                "floor_ms": alg_bytes / (pk * 1e9) * 1e3 if pk else None,
                "kernel_ms_per_launch": k_ms, "kernel_share_of_step": k_ms / (ms / a.steps),
                "dram_gbs": traffic / (k_ms * 1e-3) / 1e9 if traffic else None,
                "dram_frac": traffic / (k_ms * 1e-3) / 1e9 / peak if traffic else None,
                "traffic_note": tnote if traffic is None else tnote.get("source"),
                "union_bytes_per_launch": union_bytes,
                "union_gbs": union_bytes / (k_ms * 1e-3) / 1e9 if k_ms > 0 else None,
                "effective_gather_gbs": sl_bytes / (k_ms * 1e-3) / 1e9 if k_ms > 0 else None,
                "union_rows_per_step": avg("union_rows"), "pairs_algorithmic": total_cand,
                "pairs_kept": avg("pairs_kept"), "pairs_rescored": avg("pairs_scored") if kind == 2 else None,
                "rescore_ms": avg("ms_rescore") if kind == 2 else None,
                "k_slots": avg("k_slots") if kind == 2 else None}
        res = {
            "metric": METRIC, "value": nq * a.steps / (ms * 1e-3), "unit": UNIT, "n_gpus": world,
            "steps": a.steps, "warmup": a.warmup, "ms_per_step": ms / a.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic (seeded Gaussian mixture, torch Philox on device; synth/)",
            "config": {"workload": wl, "n": cfg.n, "d": cfg.d, "nq": nq, "k": k, "G": cfg.G, "M": cfg.M, "L": cfg.L,
                       "W": cfg.W, "probe": cfg.probe, "T": cfg.T, "hierarchy": cfg.hierarchy,
                       "parallelism": f"leaf-shard{world}" if world > 1 else "single",
                       "l2": "no flush: table (%.1f GB) and query batch (%.0f MB) exceed the 126 MB L2"
                             % (cfg.n * info.d_stride * 4 / 1e9, nq * cfg.d * 4 / 1e6)},
            "recall@10": recall, "recall_note": recall_note, "error_ratio@10": kappa,
            "leaf_ceiling@10": ceiling,
            "selectivity": total_cand / nq / cfg.n, "mean_candidates": total_cand / nq,
            "build_s": build_s, "datagen_s": gen_s,
            "roofline": roof,
            "stage_ms": {k2: avg(k2) for k2 in ("ms_route_hash", "ms_probe", "ms_plan", "ms_shortlist", "ms_screen",
                                                 "ms_rescore", "ms_merge", "ms_total")},
            "gpu_launches": launches,
            "shard_load": shard_load,
            "e2e": e2e,
            "cpu_baseline": cpu,
            "clocks": clocks,
        }
        print(json.dumps(res), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


# --- oracle arms ----------------------------------------------------------------------

def _oracle_index(cfg, Xh):
    import oracle
    t0 = time.time()
    ox = oracle.OracleIndex(Xh, G=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index, quantizer=cfg.quantizer, L=cfg.L)
    return ox, time.time() - t0


def _oracle_rate(ox, cfg, Qh, target_s, max_q=None):
    """Time the oracle's query phase on growing prefixes of the batch until ~target_s."""
    nq = Qh.shape[0]
    m = 64
    last = None
    while True:
        m = min(m, nq if max_q is None else min(nq, max_q))
        t0 = time.perf_counter()
        ox.query(Qh[:m], cfg.k, probe=cfg.probe, T=cfg.T, hierarchy=cfg.hierarchy, min_cand=cfg.min_cand)
        dt = time.perf_counter() - t0
        last = (m, dt)
        if dt >= target_s or m >= nq or (max_q is not None and m >= max_q):
            return last
        m = int(m * min(8.0, max(1.5, 1.2 * target_s / max(dt, 1e-3))))


def cpu_baseline(cfg, X, Q, target_s):
    import oracle
    Xh = X.cpu().numpy()
    Qh = Q.cpu().numpy()
    ox, bt = _oracle_index(cfg, Xh)
    m, dt = _oracle_rate(ox, cfg, Qh, target_s)
    note = ""
    if cfg.hierarchy and cfg.min_cand == 0:
        note = "; tau = median over the sample"
    return {"value": m / dt, "unit": UNIT, "cores": oracle.num_threads(), "kind": "oracle",
            "sample": f"query phase (route, hash, probe, lookup, short-list) of the first {m} queries of the "
                      f"same batch against the oracle's own index of the full dataset (build {bt:.0f}s untimed){note}"}


def run_reference(a):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import torch
    import oracle
    import synth
    cfg = load_cfg(a)
    dev = "cuda:0" if torch.cuda.is_available() else None
    if dev:
        X, Q = synth.make_dataset(cfg, backend="torch", device=dev)
        Xh, Qh = X.cpu().numpy(), Q.cpu().numpy()
        del X, Q
    else:
        Xh, Qh = synth.make_dataset(cfg, backend="numpy")
    ox, bt = _oracle_index(cfg, Xh)
    # size each step as a bounded sample: about 8 s of oracle work per step
    m, dt = _oracle_rate(ox, cfg, Qh, 8.0)
    for i in range(a.warmup):
        ox.query(Qh[:m], cfg.k, probe=cfg.probe, T=cfg.T, hierarchy=cfg.hierarchy, min_cand=cfg.min_cand)
    t0 = time.perf_counter()
    for i in range(a.steps):
        ox.query(Qh[:m], cfg.k, probe=cfg.probe, T=cfg.T, hierarchy=cfg.hierarchy, min_cand=cfg.min_cand)
    el = time.perf_counter() - t0
    v = m * a.steps / el
    res = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": int(os.environ.get("WORLD_SIZE", "1")),
           "steps": a.steps, "warmup": a.warmup, "ms_per_step": el / a.steps * 1e3, "higher_is_better": True,
           "scaling": "strong", "vs_baseline": None, "dtype": "f64",
           "data": "synthetic (seeded Gaussian mixture; synth/)",
           "config": {"workload": workload_str(cfg)},
           "cpu_baseline": {"value": v, "unit": UNIT, "kind": "oracle", "cores": oracle.num_threads(),
                            "sample": f"each step = oracle query phase on {m} queries of the batch "
                                      f"(index build {bt:.0f}s untimed)"},
           "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(res), flush=True)


def main():
    a = parse()
    if a.impl == "reference":
        run_reference(a)
    else:
        run_ours(a)


if __name__ == "__main__":
    main()
