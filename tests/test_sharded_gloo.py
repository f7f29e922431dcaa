"""N > 1 path on CPU: the leaf-sharded exchange of paper_conf_icde_panm12_b200.sharded
over a world-size-2 gloo process group.

No GPU here, so each rank's shard answers come from a stand-in built on the CPU
oracle: the oracle's full index, with the rows of queries whose leaf the rank
does not own replaced by padding (exactly what blsh_query_packed does on a
sharded index), and a numpy k-smallest merge in place of blsh_merge_topk.  What
is under test is the product's exchange logic: the leaf partition, the packed
(d^2, id) layout, the all-gather order, the SUM all-reduce of the base counts
that gives the hierarchy's global batch median (R18), and that the merged
result equals the single-index result bit for bit.
"""
import os
import socket
import tempfile

import numpy as np
import pytest

PAD = np.uint64(0x7F800000FFFFFFFF)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _pack(ids, d2):
    bits = d2.astype(np.float32).view(np.uint32).astype(np.uint64)
    out = (bits << np.uint64(32)) | (ids.astype(np.int64) & 0xFFFFFFFF).astype(np.uint64)
    out[ids < 0] = PAD
    return out


def _np_merge(gathered, n_lists, nq, k, out=None):
    g = gathered.numpy().view(np.uint64).reshape(n_lists, nq, k)
    m = np.sort(g.transpose(1, 0, 2).reshape(nq, n_lists * k), axis=1)[:, :k]
    ids = np.where(m == PAD, -1, (m & np.uint64(0xFFFFFFFF)).astype(np.int64))
    d2 = (m >> np.uint64(32)).astype(np.uint32).view(np.float32)
    return ids, d2


class _OracleShard:
    """Stand-in for a sharded blsh index (rank's leaves only), built on the oracle."""

    def __init__(self, ox, lo, hi):
        self.ox, self.lo, self.hi = ox, lo, hi

    def _owned(self, nq):
        ql = self.ox.get("q_leaf")
        assert len(ql) == nq
        return (ql >= self.lo) & (ql < self.hi)

    def base_counts(self, Q, probe=0, n_probes=1):
        import torch
        self.ox.query(Q, 1, probe=probe, T=n_probes)
        b = self.ox.get("q_base").copy()
        b[~self._owned(len(Q))] = 0
        return torch.from_numpy(b)

    def query_packed(self, Q, k, probe=0, n_probes=1, hierarchy=0, min_cand=0, global_base=None, timing=False):
        import torch
        tau = min_cand
        if hierarchy and not min_cand:
            gb = np.sort(global_base.numpy())
            tau = int(gb[(len(gb) - 1) // 2])         # lower median (R18)
        ids, d2, nc = self.ox.query(Q, k, probe=probe, T=n_probes, hierarchy=hierarchy, min_cand=tau)
        pk = _pack(ids, d2)
        own = self._owned(len(Q))
        pk[~own] = PAD
        nc = nc.copy()
        nc[~own] = 0                                  # blsh_query_packed: 0 for queries of other shards
        return torch.from_numpy(pk.view(np.int64)), torch.from_numpy(nc)


def _worker(rank, world, port, outdir, probe, T, hierarchy):
    import torch.distributed as dist
    import oracle
    import synth
    from paper_conf_icde_panm12_b200.sharded import ShardedIndex, leaf_range
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        cfg = synth.CONFIGS["c1"]
        X, Q = synth.make_dataset(cfg, n=3000, nq=96)
        ox = oracle.OracleIndex(X, G=4, M=8, W=4.0, seed=11)
        lo, hi = leaf_range(4, rank, world)
        sh = ShardedIndex(_OracleShard(ox, lo, hi), merge=_np_merge)
        ids, d2 = sh.query(Q, 10, probe=probe, n_probes=T, hierarchy=hierarchy)
        if hierarchy:
            gb = sh.global_base_counts(Q, probe, T).numpy()
            np.save(os.path.join(outdir, f"gb{rank}.npy"), gb)
        np.save(os.path.join(outdir, f"load{rank}.npy"), np.array(sh.load_stats(), np.int64))
        np.save(os.path.join(outdir, f"ids{rank}.npy"), ids)
        np.save(os.path.join(outdir, f"d2{rank}.npy"), d2)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("probe,T,hierarchy", [(0, 1, 0), (1, 16, 0), (0, 1, 1), (1, 8, 1)])
def test_sharded_exchange_equals_single_index(orc, probe, T, hierarchy):
    import torch.multiprocessing as mp
    import synth
    world = 2
    with tempfile.TemporaryDirectory() as td:
        mp.spawn(_worker, args=(world, _free_port(), td, probe, T, hierarchy), nprocs=world, join=True)
        cfg = synth.CONFIGS["c1"]
        X, Q = synth.make_dataset(cfg, n=3000, nq=96)
        ox = orc.OracleIndex(X, G=4, M=8, W=4.0, seed=11)
        ids_ref, d2_ref, nc_ref = ox.query(Q, 10, probe=probe, T=T, hierarchy=hierarchy)
        if hierarchy:
            base_ref = ox.get("q_base")
        for r in range(world):
            ids = np.load(os.path.join(td, f"ids{r}.npy"))
            d2 = np.load(os.path.join(td, f"d2{r}.npy"))
            assert np.array_equal(ids, ids_ref), f"rank {r}: merged ids differ from the single index"
            assert np.array_equal(d2.view(np.uint32), d2_ref.view(np.uint32)), f"rank {r}: merged d2 differ"
            if hierarchy:
                assert np.array_equal(np.load(os.path.join(td, f"gb{r}.npy")), base_ref)
            # per-rank load (all-gathered, the same on every rank): the shards split the batch's work
            load = np.load(os.path.join(td, f"load{r}.npy"))
            assert load.shape == (world, 2)
            assert load[:, 0].sum() == int((nc_ref > 0).sum()) and load[:, 1].sum() == int(nc_ref.sum())
            assert np.array_equal(load, np.load(os.path.join(td, "load0.npy")))
        # the exchange was not vacuous: both shards own queries
        ql = ox.get("q_leaf")
        assert 0 < int((ql < 2).sum()) < len(ql)


def test_leaf_range_partition():
    from paper_conf_icde_panm12_b200.sharded import leaf_range
    for G, P in [(64, 8), (64, 1), (16, 4), (4, 2)]:
        got = [leaf_range(G, r, P) for r in range(P)]
        assert got[0][0] == 0 and got[-1][1] == G
        assert all(got[i][1] == got[i + 1][0] for i in range(P - 1))
        assert len({h - l for l, h in got}) == 1
    with pytest.raises(ValueError):
        leaf_range(64, 0, 3)


def test_balanced_leaf_split_is_optimal():
    """balanced_leaf_split = the best contiguous partition (brute force over all of them)."""
    import itertools
    from paper_conf_icde_panm12_b200.sharded import balanced_leaf_split
    rng = np.random.default_rng(2)
    for _ in range(60):
        G = int(rng.integers(1, 9))
        world = int(rng.integers(1, 5))
        w = rng.integers(0, 50, G).tolist()
        b = balanced_leaf_split(w, world)
        assert len(b) == world + 1 and b[0] == 0 and b[-1] == G and all(x <= y for x, y in zip(b, b[1:]))
        got = max(sum(w[b[r]:b[r + 1]]) for r in range(world))
        best = None
        for cuts in itertools.combinations_with_replacement(range(G + 1), world - 1):
            bb = [0, *cuts, G]
            m = max(sum(w[bb[r]:bb[r + 1]]) for r in range(world))
            best = m if best is None else min(best, m)
        assert got == best
    # a skewed batch: the hot leaf gets a rank of its own
    assert balanced_leaf_split([100, 1, 1, 1, 1, 1, 1, 1], 2) == [0, 1, 8]
