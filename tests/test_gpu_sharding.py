"""Load-aware leaf -> rank assignment: shards built with a
`leaf_split` from balanced_leaf_split over measured per-leaf loads answer
exactly like one GPU, including world sizes that do not divide G."""
import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def blsh():
    if not torch.cuda.is_available():
        pytest.skip("needs CUDA")
    from paper_conf_icde_panm12_b200 import blsh as b
    b.lib()
    return b


@pytest.mark.parametrize("G,world", [(4, 3), (8, 2), (8, 5)])
def test_leaf_split_shards_match_single(blsh, G, world):
    from paper_conf_icde_panm12_b200.sharded import balanced_leaf_split
    X, Q = synth.make_dataset(synth.CONFIGS["c1"])
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    full = blsh.blsh_build(Xd, n_leaves=G, M=8, W=4.0, seed=42)
    i1, d1, n1 = full.query(Qd, 10, probe=1, n_probes=8, keep_stages=True)
    leaf, base = full.export("Q_LEAF"), full.export("Q_BASE")
    loads = np.bincount(leaf, weights=base.astype(np.float64), minlength=G).astype(np.int64)
    split = balanced_leaf_split(loads, world)
    parts, ncs, owned = [], [], []
    for r in range(world):
        sh = blsh.blsh_build(Xd, n_leaves=G, M=8, W=4.0, seed=42, rank=r, world=world, leaf_split=split)
        info = sh.info()
        assert (info.leaf_lo, info.leaf_hi) == (split[r], split[r + 1])
        pk, nc = sh.query_packed(Qd, 10, probe=1, n_probes=8)
        parts.append(pk)
        ncs.append(nc)
        owned.append(int(info.n_owned))
    mi, md = blsh.blsh_merge_topk(torch.cat(parts).contiguous(), world, len(Q), 10)
    torch.cuda.synchronize()
    assert torch.equal(mi, i1) and torch.equal(md.view(torch.int32), d1.view(torch.int32))
    assert torch.equal(sum(ncs), n1)
    assert sum(owned) == len(X)
    # the largest shard load is the optimum of the contiguous partitions
    got = max(int(loads[split[r]:split[r + 1]].sum()) for r in range(world))
    assert got <= int(np.ceil(loads.sum() / world)) + int(loads.max())


def test_leaf_split_validation(blsh):
    X, _ = synth.make_dataset(synth.CONFIGS["c1"])
    Xd = torch.from_numpy(X).cuda()
    with pytest.raises(blsh.BlshError):
        blsh.blsh_build(Xd, n_leaves=4, rank=0, world=3)                          # 3 does not divide 4
    with pytest.raises(blsh.BlshError):
        blsh.blsh_build(Xd, n_leaves=4, rank=0, world=2, leaf_split=[0, 3, 2])    # decreasing
    with pytest.raises(blsh.BlshError):
        blsh.blsh_build(Xd, n_leaves=4, rank=0, world=2, leaf_split=[1, 2, 4])    # not from 0


@pytest.mark.parametrize("G,L", [(4, 1), (8, 1), (4, 3)])
def test_w_rule_parity(blsh, orc, G, L):
    """W_rule = 1 (R29): per-leaf widths, redrawn (a, b), tables and queries bit-exact."""
    from parity_utils import check_topk
    X, Q = synth.make_dataset(synth.CONFIGS["c1"])
    ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=G, M=8, W=3.0, seed=5, W_rule=1, n_tables=L,
                         keep_stages=True)
    ox = orc.OracleIndex(X, G=G, M=8, W=3.0, seed=5, W_rule=1, L=L)
    assert np.array_equal(ix.export("W").view(np.uint32), ox.get("W").view(np.uint32)), "per-leaf W differs"
    assert len(set(ix.export("W").tolist())) > 1
    for l in range(L):
        for a, b in [("A", "A"), ("B", "b"), ("PERM", "perm"), ("UKEY", "ukey"), ("UOFF", "uoff")]:
            assert np.array_equal(ix.export(a, table=l).view(np.uint8), ox.get(b, l).ravel().view(np.uint8)), a
    ids, d2, nc = ix.query(torch.from_numpy(Q).cuda(), 10, probe=1, n_probes=8)
    torch.cuda.synchronize()
    oi, od, onc = ox.query(Q, 10, probe=1, T=8)
    assert np.array_equal(nc.cpu().numpy(), onc)
    check_topk(ids.cpu().numpy(), d2.cpu().numpy(), oi, od, X, Q, cands=ox.candidates())
