"""Seeded synthetic inputs for Bi-level LSH (shared by the oracle side and the CUDA side).

This module holds NO arithmetic of the method (no hashing, no tree, no
distances): it only draws data points and queries, and names the benchmark
configurations.  Both the CPU oracle (``oracle/``) and the CUDA library
(``paper_conf_icde_panm12_b200/``) consume what it produces; neither imports
the other.

Workload shape: Gaussian
mixtures shaped like the paper's GIST image features (LabelMe 512-d,
Tiny Images 384-d), with low intrinsic dimension (the RP-tree premise)::

    centre  mu_c ~ N(0, I_d)
    basis   B_c  in R^{d x r}, entries N(0, spread^2 / r)
    point   x = mu_c + B_c z + 0.01 * spread * eps,   z ~ N(0, I_r), eps ~ N(0, I_d)

Queries are a disjoint sample of the same mixture, optionally with
a fraction of "between-cluster" queries (midpoint of two centres + noise) that
land in low-density regions.

Two backends draw the same recipe: ``numpy`` (PCG64; CPU tests and small GPU
parity cases) and ``torch`` (Philox on a CUDA device; benchmark-scale data that
would take minutes to draw on the host).  They produce different numbers for
the same seed; a configuration states which backend it uses.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field, replace
from typing import Optional

import numpy as np

__all__ = ["Config", "CONFIGS", "mixture", "sample_points", "sample_queries", "make_dataset"]


@dataclass(frozen=True)
class Config:
    """One workload of BASELINE.json ``configs`` (index = position there, 1-based)."""

    name: str
    n: int
    d: int
    n_clusters: int
    spread: float
    rank: int
    nq: int
    k: int
    G: int
    M: int
    W: float
    probe: int = 0            # 0 standard, 1 multiprobe, 2 lattice (E8)
    T: int = 1
    hierarchy: int = 0
    min_cand: int = 0
    quantizer: int = 0        # 0 Z^M floor, 1 E8
    L: int = 1                # hash tables per leaf
    zipf: float = 0.0
    between: float = 0.0
    backend: str = "numpy"
    seed_data: int = 1001
    seed_query: int = 2001
    seed_index: int = 42
    notes: str = ""


# W values are absolute (data units).  They were chosen by the calibration
# sweep in tools/calibrate.py: the smallest
# selectivity meeting recall@10 >= 0.9 among W in r10 * {2, 2.83, 4, 5.66, 8}.
CONFIGS = {
    "c1": Config("c1", n=10_000, d=64, n_clusters=16, spread=0.05, rank=64, nq=100, k=10,
                 G=4, M=8, W=4.0, seed_data=1001, seed_query=2001,
                 notes="BASELINE configs[0]: CPU-oracle-in-seconds case"),
    "c2": Config("c2", n=22_000, d=512, n_clusters=64, spread=0.02, rank=16, nq=1_000, k=50,
                 G=4, M=8, W=7.03, L=4, seed_data=1002, seed_query=2002,
                 notes="BASELINE configs[1]: LabelMe-shaped, standard LSH per subgroup (L = 4 tables); "
                       "G = 4, W = 16 r10 (calibrated r02ai: recall@10 0.953, leaf ceiling 0.963)"),
    "c3": Config("c3", n=1_000_000, d=384, n_clusters=256, spread=0.02, rank=16, nq=10_000,
                 k=50, G=8, M=8, W=2.41, probe=1, T=16, hierarchy=1, min_cand=0, zipf=0.8,
                 between=0.05, backend="torch", seed_data=1003, seed_query=2003,
                 notes="BASELINE configs[2]: Tiny-Images-shaped, multiprobe + Morton hierarchy; "
                       "G = 8, W = 8 r10 (calibrated r02ah: recall@10 0.922, leaf ceiling 0.935)"),
    "c4": Config("c4", n=10_000_000, d=384, n_clusters=1024, spread=0.02, rank=16,
                 nq=100_000, k=10, G=64, M=8, W=2.33, probe=1, T=16, backend="torch",
                 seed_data=1004, seed_query=2004,
                 notes="BASELINE configs[3]: 10M x 384 sharded by subgroup, NCCL top-k merge; "
                       "W = 8 r10, T = 16 (recalibrated r02ai under the fp16 screen: recall@10 0.930)"),
    "c5": Config("c5", n=1_000_000, d=384, n_clusters=256, spread=0.02, rank=16, nq=100_000,
                 k=10, G=16, M=8, W=2.51, probe=1, T=16, backend="torch",
                 seed_data=1005, seed_query=2005,
                 notes="BASELINE configs[4]: sweep base (probes 1-64, lattice vs multiprobe, batch)"),
    # The paper's own evaluation setting: 100,000 items hashed, another
    # 100,000 items of the same distribution as queries, L = 10 tables, M = 8,
    # k = 500 (Tiny-Images-shaped 384-d data).
    "p217": Config("p217", n=100_000, d=384, n_clusters=64, spread=0.02, rank=16, nq=100_000,
                   k=500, G=16, M=8, W=1.90, probe=0, T=1, L=10, backend="torch",
                   seed_data=1006, seed_query=2006,
                   notes="P:217 evaluation setting: L = 10, M = 8, k = 500, 100k items / 100k queries; "
                         "W = 5.66 r10 (calibrated r02aj: recall@10 0.911, leaf ceiling 0.937)"),
}


@dataclass
class Mixture:
    centres: np.ndarray      # [C, d]
    bases: np.ndarray        # [C, d, r]
    weights: np.ndarray      # [C]
    spread: float


def _weights(C: int, zipf: float) -> np.ndarray:
    if zipf <= 0.0:
        return np.full(C, 1.0 / C)
    w = 1.0 / np.arange(1, C + 1, dtype=np.float64) ** zipf
    return w / w.sum()


def mixture(d: int, C: int, rank: int, spread: float, seed: int, zipf: float = 0.0) -> Mixture:
    """Mixture parameters (always numpy, small); stream 0 of ``seed``."""
    rng = np.random.default_rng([seed, 0])
    centres = rng.standard_normal((C, d))
    bases = rng.standard_normal((C, d, rank)) * (spread / math.sqrt(rank))
    return Mixture(centres, bases, _weights(C, zipf), spread)


def _counts(rng: np.random.Generator, n: int, w: np.ndarray) -> np.ndarray:
    return rng.multinomial(n, w)


def sample_points(mix: Mixture, n: int, seed: int, stream: int = 1, backend: str = "numpy",
                  device: Optional[str] = None):
    """n points of the mixture, fp32 row-major, in a random (seeded) order.

    backend="numpy" returns np.ndarray; backend="torch" returns a torch tensor
    on ``device`` (default cuda:0)."""
    C, d, r = mix.bases.shape
    rng = np.random.default_rng([seed, stream])
    counts = _counts(rng, n, mix.weights)
    if backend == "numpy":
        out = np.empty((n, d), dtype=np.float32)
        pos = 0
        for c in range(C):
            m = int(counts[c])
            if m == 0:
                continue
            z = rng.standard_normal((m, r))
            eps = rng.standard_normal((m, d))
            x = mix.centres[c] + z @ mix.bases[c].T + (0.01 * mix.spread) * eps
            out[pos:pos + m] = x.astype(np.float32)
            pos += m
        perm = rng.permutation(n)
        return out[perm]
    if backend == "torch":
        import torch
        dev = torch.device(device or "cuda:0")
        gen = torch.Generator(device=dev)
        gen.manual_seed(int(seed) * 1_000_003 + int(stream))
        centres = torch.as_tensor(mix.centres, dtype=torch.float32, device=dev)
        bases = torch.as_tensor(mix.bases, dtype=torch.float32, device=dev)
        out = torch.empty((n, d), dtype=torch.float32, device=dev)
        pos = 0
        for c in range(C):
            m = int(counts[c])
            if m == 0:
                continue
            z = torch.randn((m, r), generator=gen, device=dev)
            blk = out[pos:pos + m]
            torch.randn((m, d), generator=gen, device=dev, out=blk)
            blk.mul_(0.01 * mix.spread)
            blk.add_(z @ bases[c].T)
            blk.add_(centres[c])
            pos += m
        perm = torch.randperm(n, generator=gen, device=dev)
        return out[perm].contiguous()
    raise ValueError(f"unknown backend {backend!r}")


def sample_queries(mix: Mixture, nq: int, seed: int, between: float = 0.0, backend: str = "numpy",
                   device: Optional[str] = None):
    """Queries: a disjoint sample of the same mixture; a fraction
    ``between`` are midpoints of two random centres plus noise."""
    q = sample_points(mix, nq, seed, stream=1, backend=backend, device=device)
    nb = int(round(between * nq))
    if nb == 0:
        return q
    C, d, _ = mix.bases.shape
    rng = np.random.default_rng([seed, 2])
    a = rng.integers(0, C, size=nb)
    b = (a + 1 + rng.integers(0, C - 1, size=nb)) % C
    mid = 0.5 * (mix.centres[a] + mix.centres[b]) + mix.spread * rng.standard_normal((nb, d))
    idx = rng.choice(nq, size=nb, replace=False)
    if backend == "numpy":
        q[idx] = mid.astype(np.float32)
        return q
    import torch
    q[torch.as_tensor(idx, device=q.device)] = torch.as_tensor(mid, dtype=torch.float32, device=q.device)
    return q


def make_dataset(cfg: Config, n: Optional[int] = None, nq: Optional[int] = None,
                 backend: Optional[str] = None, device: Optional[str] = None):
    """(X, Q) for a configuration; n / nq / backend override the config's."""
    be = backend or cfg.backend
    mix = mixture(cfg.d, cfg.n_clusters, cfg.rank, cfg.spread, cfg.seed_data, cfg.zipf)
    X = sample_points(mix, n or cfg.n, cfg.seed_data, stream=1, backend=be, device=device)
    Q = sample_queries(mix, nq or cfg.nq, cfg.seed_query, cfg.between, backend=be, device=device)
    return X, Q


def small(cfg: Config, **kw) -> Config:
    """A reduced copy of a configuration (for tests)."""
    return replace(cfg, **kw)
