"""Leaf-sharded multi-GPU query path (a6).

The RP-tree's first level is a hard partition (a query only ever touches
its own leaf), so the index shards by leaf: rank r of P keeps leaves
[r*G/P, (r+1)*G/P) (``blsh_build(..., rank, world)``; the tree and parameters
are rebuilt identically from the seed on every rank).  A query batch goes to
every rank; each rank answers the queries of its own leaves and pads the rest
(``blsh_query_packed``), the per-rank packed (d^2, id) lists are exchanged with
ONE all-gather over NVLink / NVSwitch (NCCL) and ``blsh_merge_topk`` keeps the
k smallest per query.  Every query has exactly one owner, so the merged result
is bit-identical to the single-GPU result.

The Morton hierarchy's batch-median threshold (R18) is a statistic of the
whole batch; on a sharded index it needs the base counts |A0(q)| of every query:
``blsh_query_base_counts`` on each rank (0 for queries it does not own) and a
SUM all-reduce give exactly the single-GPU counts, passed to the query as
``global_base``.

This module is process-group plumbing only (torch.distributed); all arithmetic
runs in libblsh.so.  ``index`` and ``merge`` can be swapped for stand-ins so the
exchange logic is testable on CPU with the gloo backend (tests/test_sharded_gloo.py).
"""
from __future__ import annotations

from typing import Callable, Optional


def leaf_range(G: int, rank: int, world: int):
    """Leaves owned by `rank` (mirrors blsh_build's partition; world must divide G)."""
    if world < 1 or not 0 <= rank < world or G % world:
        raise ValueError("need 0 <= rank < world and world | G")
    per = G // world
    return rank * per, (rank + 1) * per


def balanced_leaf_split(weights, world: int):
    """Load-aware leaf -> rank assignment (query skew across leaves):
    the contiguous partition of the leaves into `world` ranges whose largest load
    sum is minimal (binary search on that bound + greedy fill).  Returns the
    [world + 1] boundaries blsh_build takes as `leaf_split`."""
    w = [int(x) for x in weights]
    if world < 1 or any(x < 0 for x in w):
        raise ValueError("need world >= 1 and non-negative weights")
    G = len(w)

    def ranges_needed(cap):
        n, acc = 1, 0
        for x in w:
            if acc + x > cap:
                n, acc = n + 1, x
            else:
                acc += x
        return n

    lo, hi = max(w) if w else 0, sum(w)
    while lo < hi:
        mid = (lo + hi) // 2
        if ranges_needed(mid) <= world:
            hi = mid
        else:
            lo = mid + 1
    bounds, acc = [0], 0
    for g, x in enumerate(w):
        if acc + x > lo and len(bounds) < world:
            bounds.append(g)
            acc = x
        else:
            acc += x
    while len(bounds) < world:
        bounds.append(G)
    bounds.append(G)
    return bounds


class ShardedIndex:
    """One leaf shard of a Bi-level LSH index per process of `group`."""

    def __init__(self, index, group=None, merge: Optional[Callable] = None):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.index = index
        if merge is None:
            from . import blsh
            merge = blsh.blsh_merge_topk
        self._merge = merge
        self._gathered = None
        self.last_ncand = None

    @classmethod
    def build(cls, X, group=None, **build_kw) -> "ShardedIndex":
        import torch.distributed as dist
        from . import blsh
        ix = blsh.blsh_build(X, rank=dist.get_rank(group), world=dist.get_world_size(group), **build_kw)
        return cls(ix, group)

    def global_base_counts(self, Q, probe: int = 0, n_probes: int = 1, curve_perturb: int = 0):
        """|A0(q)| of every query of the batch over all shards (SUM all-reduce of the per-rank counts)."""
        import torch
        kw = {}
        if not (isinstance(Q, torch.Tensor) and Q.is_cuda) and torch.cuda.is_available():
            kw["out"] = torch.empty((int(Q.shape[0]),), dtype=torch.int64, device="cuda")   # all-reduce on device
        if curve_perturb:
            kw["curve_perturb"] = curve_perturb
        base = self.index.base_counts(Q, probe=probe, n_probes=n_probes, **kw)
        if self.world > 1:
            self.dist.all_reduce(base, op=self.dist.ReduceOp.SUM, group=self.group)
        return base

    def leaf_loads(self, Q, k: int, **kw):
        """Per-leaf work of a (sample) batch on the whole sharded index: sum of |A(q)| over
        the queries routed to each leaf (this rank's leaves from its own answers, the rest
        from the other ranks: SUM all-reduce).  Feeds balanced_leaf_split."""
        import numpy as np
        import torch
        self.index.query_packed(Q, k, keep_stages=True, **kw)
        leaf = self.index.export("Q_LEAF")
        nc = self.index.export("Q_BASE") if not kw.get("hierarchy") else None
        if nc is None:
            raise ValueError("leaf_loads: use a probe configuration without the hierarchy")
        G = int(self.index.info().G)
        loads = np.bincount(leaf, weights=nc.astype(np.float64), minlength=G).astype(np.int64)
        t = torch.from_numpy(loads)
        if torch.cuda.is_available():
            t = t.cuda()
        if self.world > 1:
            self.dist.all_reduce(t, op=self.dist.ReduceOp.SUM, group=self.group)
        return t.cpu().numpy()

    def load_stats(self, ncand=None):
        """Per-rank load of the last query (SURVEY §8(e) scaling risk: query skew across
        leaves): [[queries with candidates, sum |A(q)|] for every rank], all-gathered."""
        import torch
        nc = self.last_ncand if ncand is None else ncand
        mine = torch.stack([(nc > 0).sum(), nc.sum()]).to(torch.int64)
        if self.world == 1:
            return [mine.tolist()]
        allv = [torch.empty_like(mine) for _ in range(self.world)]
        self.dist.all_gather(allv, mine, group=self.group)
        return [v.tolist() for v in allv]

    def query(self, Q, k: int, out=None, timing: bool = False, packed_out=None, **kw):
        """-> (ids [nq,k] int64, dist2 [nq,k] fp32): the merged top-k of the whole sharded index.

        packed_out: optional DEVICE buffers (packed [nq,k] int64, ncand [nq] int64) for this
        rank's list; required when Q is a host array (the all-gather runs on device memory)."""
        import torch
        nq = int(Q.shape[0])
        if kw.get("hierarchy") == 1 and not kw.get("min_cand") and kw.get("global_base") is None:
            kw["global_base"] = self.global_base_counts(Q, kw.get("probe", 0), kw.get("n_probes", 1),
                                                        kw.get("curve_perturb", 0))
        if packed_out is not None:
            kw["out"] = packed_out
        pk, nc = self.index.query_packed(Q, k, timing=timing, **kw)
        self.last_ncand = nc
        if self.world == 1:
            return self._merge(pk, 1, nq, k, out=out)
        shape = (self.world * nq, k)
        if self._gathered is None or tuple(self._gathered.shape) != shape or self._gathered.device != pk.device:
            self._gathered = torch.empty(shape, dtype=pk.dtype, device=pk.device)
        # [world][nq][k] in rank order: the layout blsh_merge_topk expects
        self.dist.all_gather_into_tensor(self._gathered, pk, group=self.group)
        return self._merge(self._gathered, self.world, nq, k, out=out)
