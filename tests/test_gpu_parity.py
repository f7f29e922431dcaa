"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bit-exact: parameters, tree, per-point leaf/code/key, table, per-query
leaf/t/code/key/probe keys/candidate sets.  Distances within 1e-5 relative,
ids equal except ties (parity_utils.check_topk).
"""
import os

import numpy as np
import pytest

import synth
from parity_utils import check_topk, gpu_candidates

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def blsh():
    if not torch.cuda.is_available():
        pytest.skip("needs CUDA")
    from paper_conf_icde_panm12_b200 import blsh as b
    b.lib()
    return b


def build_pair(blsh, orc, X, G, M=8, W=4.0, seed=42, quantizer=0, device=True, **kw):
    Xin = torch.from_numpy(X).cuda() if device else X
    ix = blsh.blsh_build(Xin, n_leaves=G, M=M, W=W, seed=seed, quantizer=quantizer, keep_stages=True, **kw)
    okw = {kk: v for kk, v in kw.items() if kk in ("rp_rule", "rp_mean_c", "rp_max_jitter", "ek_iters", "W_leaf")}
    ox = orc.OracleIndex(X, G=G, M=M, W=W, seed=seed, quantizer=quantizer, **okw)
    return ix, ox


def compare_build(ix, ox, owned_all=True):
    G = ox.G
    for a, b in [("A", "A"), ("B", "b"), ("W", "W"), ("DIRS", "dirs"), ("THETA", "theta"), ("NTYPE", "ntype"),
                 ("MU", "mu"), ("DIAM2", "diam2"), ("DA2", "da2")]:
        g = ix.export(a)
        o = ox.get(b).ravel()
        assert g.shape == o.shape and np.array_equal(g.view(np.uint8), o.view(np.uint8)), f"{a} differs"
    assert np.array_equal(ix.export("POINT_LEAF"), ox.get("leaf")), "point leaf differs"
    if owned_all:
        assert np.array_equal(ix.export("POINT_CODE"), ox.get("code").ravel()), "point codes differ"
        assert np.array_equal(ix.export("POINT_KEY"), ox.get("key").ravel()), "point keys differ"
        assert np.array_equal(ix.export("PERM"), ox.get("perm")), "perm differs"
        assert np.array_equal(ix.export("UKEY"), ox.get("ukey").ravel()), "bucket keys differ"
        assert np.array_equal(ix.export("ULEAF"), ox.get("uleaf")), "bucket leaves differ"
        assert np.array_equal(ix.export("UOFF"), ox.get("uoff")), "bucket offsets differ"
        assert np.array_equal(ix.export("LEAF_U"), ox.get("leaf_u")), "leaf bucket ranges differ"


def run_query_pair(ix, ox, X, Q, k, probe=0, T=1, hierarchy=0, hier_step_bits=0, min_cand=0, device=True,
                   check_stages=True, **extra):
    """extra: curve_perturb / msb_min (R31/R32), passed to both sides."""
    Qin = torch.from_numpy(Q).cuda() if device else Q
    ids, d2, nc = ix.query(Qin, k, probe=probe, n_probes=T, hierarchy=hierarchy, hier_step_bits=hier_step_bits,
                           min_cand=min_cand, keep_stages=True, **extra)
    if device:
        torch.cuda.synchronize()
        ids, d2, nc = ids.cpu().numpy(), d2.cpu().numpy(), nc.cpu().numpy()
    oi, od, onc = ox.query(Q, k, probe=probe, T=T, hierarchy=hierarchy, hier_step_bits=hier_step_bits,
                           min_cand=min_cand, **extra)
    if check_stages:
        assert np.array_equal(ix.export("Q_LEAF"), ox.get("q_leaf")), "query leaf differs"
        assert np.array_equal(ix.export("Q_T").view(np.uint32), ox.get("q_t").ravel().view(np.uint32)), "t differs"
        assert np.array_equal(ix.export("Q_CODE"), ox.get("q_code").ravel()), "query code differs"
        assert np.array_equal(ix.export("Q_OOR"), ox.get("q_oor")), "out-of-range flags differ"
        assert np.array_equal(ix.export("Q_KEY"), ox.get("q_key").ravel()), "query key differs"
        assert np.array_equal(ix.export("Q_PVALID"), ox.get("q_pvalid").ravel()), "probe validity differs"
        assert np.array_equal(ix.export("Q_PKEY"), ox.get("q_pkey").ravel()), "probe keys (sequence) differ"
        assert np.array_equal(ix.export("Q_BASE"), ox.get("q_base")), "|A0| differs"
        if hierarchy:
            assert np.array_equal(ix.export("Q_LEVEL"), ox.get("q_level")), "hierarchy level differs"
            assert int(ix.export("Q_TAU")[0]) == ox.tau, "tau differs"
    gc = gpu_candidates(ix, T)
    oc = ox.candidates()
    for q in range(len(Q)):
        assert np.array_equal(gc[q], oc[q]), f"candidate set of query {q} differs"
    assert np.array_equal(nc, onc)
    check_topk(ids, d2, oi, od, X, Q, cands=oc)
    if len(Q) <= 128 and k <= 64 and device and "BLSH_SHORTLIST" not in os.environ:
        # small batches default to the warp short-list: the tiled tensor-core path must
        # return the same bits on them (the large-batch product path)
        os.environ["BLSH_SHORTLIST"] = "tc"
        try:
            i2, d22, n2 = ix.query(Qin, k, probe=probe, n_probes=T, hierarchy=hierarchy,
                                   hier_step_bits=hier_step_bits, min_cand=min_cand, **extra)
            torch.cuda.synchronize()
        finally:
            del os.environ["BLSH_SHORTLIST"]
        assert np.array_equal(i2.cpu().numpy(), ids) and np.array_equal(d22.cpu().numpy().view(np.uint32), d2.view(np.uint32))
        assert np.array_equal(n2.cpu().numpy(), nc)
    return ids, d2, nc


@pytest.fixture(scope="module")
def c1():
    return synth.make_dataset(synth.CONFIGS["c1"])


@pytest.fixture(scope="module")
def c1_pair(blsh, orc, c1):
    X, _ = c1
    return build_pair(blsh, orc, X, G=4, M=8, W=4.0, seed=42)


def test_c1_build_bitexact(c1_pair):
    compare_build(*c1_pair)


@pytest.mark.parametrize("k", [1, 10, 50, 64])
def test_c1_standard(c1_pair, c1, k):
    X, Q = c1
    run_query_pair(*c1_pair, X, Q, k)


@pytest.mark.parametrize("T", [2, 16, 64, 240])
def test_c1_multiprobe(c1_pair, c1, T):
    X, Q = c1
    run_query_pair(*c1_pair, X, Q, 10, probe=1, T=T)


@pytest.mark.parametrize("step,tau", [(0, 0), (0, 300), (1, 0), (8, 5000)])
def test_c1_hierarchy(c1_pair, c1, step, tau):
    X, Q = c1
    run_query_pair(*c1_pair, X, Q, 10, probe=1, T=4, hierarchy=1, hier_step_bits=step, min_cand=tau)
    run_query_pair(*c1_pair, X, Q, 10, probe=0, T=1, hierarchy=1, hier_step_bits=step, min_cand=tau)


@pytest.mark.parametrize("T", [1, 16, 241])
def test_c1_e8_lattice(blsh, orc, c1, T):
    X, Q = c1
    ix, ox = build_pair(blsh, orc, X, G=4, M=8, W=4.0, seed=42, quantizer=1)
    compare_build(ix, ox)
    run_query_pair(ix, ox, X, Q, 10, probe=2 if T > 1 else 0, T=T)


def test_host_buffers_match_device(blsh, orc, c1):
    X, Q = c1
    ix, ox = build_pair(blsh, orc, X, G=4, device=False)
    compare_build(ix, ox)
    i1, d1, n1 = run_query_pair(ix, ox, X, Q, 10, probe=1, T=8, device=False)
    i2, d2, n2 = run_query_pair(ix, ox, X, Q, 10, probe=1, T=8, device=True)
    assert np.array_equal(i1, i2) and np.array_equal(d1, d2) and np.array_equal(n1, n2)


@pytest.mark.parametrize("G,M,W,d", [(1, 8, 2.0, 64), (8, 4, 1.5, 61), (16, 10, 3.0, 33), (2, 3, 0.5, 5),
                                     (4, 16, 6.0, 64), (32, 8, 4.0, 64)])
def test_shapes(blsh, orc, G, M, W, d):
    rng = np.random.default_rng(G * 100 + M)
    mix = synth.mixture(d, 8, min(8, d), 0.3, 77)
    X = synth.sample_points(mix, 3000, 78)
    Q = synth.sample_points(mix, 40, 79)
    ix, ox = build_pair(blsh, orc, X, G=G, M=M, W=W, seed=int(rng.integers(1, 1000)))
    compare_build(ix, ox)
    run_query_pair(ix, ox, X, Q, 10)
    if M <= 10:
        run_query_pair(ix, ox, X, Q, 7, probe=1, T=min(3 ** M, 20), hierarchy=1)
    else:
        run_query_pair(ix, ox, X, Q, 7, hierarchy=1, hier_step_bits=3)


def test_edge_cases(blsh, orc):
    rng = np.random.default_rng(5)
    # n < G (empty leaves), duplicates, all-equal points
    X = rng.standard_normal((5, 12)).astype(np.float32)
    Q = rng.standard_normal((6, 12)).astype(np.float32)
    ix, ox = build_pair(blsh, orc, X, G=16, M=4, W=1.0)
    compare_build(ix, ox)
    run_query_pair(ix, ox, X, Q, 10, probe=1, T=9, hierarchy=1)
    X = np.repeat(rng.standard_normal((1, 16)).astype(np.float32), 700, axis=0)
    ix, ox = build_pair(blsh, orc, X, G=4, M=8, W=1.0)
    compare_build(ix, ox)
    run_query_pair(ix, ox, X, X[:5].copy(), 10)
    X = rng.standard_normal((400, 16)).astype(np.float32)
    X = np.concatenate([X, X[:100]])
    ix, ox = build_pair(blsh, orc, X, G=8, M=6, W=0.8)
    compare_build(ix, ox)
    run_query_pair(ix, ox, X, X[::7].copy(), 20, probe=1, T=30)
    # d = 1
    X = rng.standard_normal((900, 1)).astype(np.float32)
    ix, ox = build_pair(blsh, orc, X, G=4, M=2, W=0.1)
    compare_build(ix, ox)
    run_query_pair(ix, ox, X, rng.standard_normal((30, 1)).astype(np.float32), 5, probe=1, T=5)


def test_sphere_split_and_max_rule(blsh, orc):
    rng = np.random.default_rng(2)
    n, d = 4000, 24
    X = (0.1 * rng.standard_normal((n, d))).astype(np.float32)
    out = rng.choice(n, 20, replace=False)
    X[out] += (40.0 * rng.standard_normal((20, d))).astype(np.float32)
    Q = np.concatenate([X[out[:5]] + 0.01, X[:20]]).astype(np.float32)
    ix, ox = build_pair(blsh, orc, X, G=4, M=4, W=1.0, seed=3)
    assert ox.get("ntype")[0] == 1
    compare_build(ix, ox)
    run_query_pair(ix, ox, X, Q, 5, probe=1, T=10)
    ix, ox = build_pair(blsh, orc, X, G=4, M=4, W=1.0, seed=3, rp_rule=1, rp_max_jitter=6.0)
    compare_build(ix, ox)
    run_query_pair(ix, ox, X, Q, 5)
    ix, ox = build_pair(blsh, orc, X, G=4, M=4, W=1.0, seed=3, ek_iters=3, rp_mean_c=1.5)
    compare_build(ix, ox)


def test_per_leaf_width(blsh, orc, c1):
    X, Q = c1
    ix, ox = build_pair(blsh, orc, X, G=4, M=8, W=4.0, W_leaf=[2.0, 3.0, 5.0, 8.0])
    compare_build(ix, ox)
    run_query_pair(ix, ox, X, Q, 10, probe=1, T=8)


def test_out_of_range_build_error(blsh):
    X = np.random.default_rng(0).standard_normal((500, 8)).astype(np.float32) * 1e4
    with pytest.raises(blsh.BlshError) as e:
        blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=2, M=8, W=1e-3)
    assert e.value.status == blsh.BLSH_ERR_RANGE


def test_invalid_args(blsh, c1):
    X, Q = c1
    ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=4)
    Qd = torch.from_numpy(Q).cuda()
    for kw, st in [(dict(k=0), blsh.BLSH_ERR_INVALID), (dict(k=1025), blsh.BLSH_ERR_UNSUPPORTED),
                   (dict(k=5, probe=2, n_probes=4), blsh.BLSH_ERR_INVALID),
                   (dict(k=5, probe=0, n_probes=4), blsh.BLSH_ERR_INVALID),
                   (dict(k=5, probe=1, n_probes=300), blsh.BLSH_ERR_UNSUPPORTED)]:
        k = kw.pop("k")
        with pytest.raises(blsh.BlshError) as e:
            ix.query(Qd, k, **kw)
        assert e.value.status == st
    ids, d2, nc = ix.query(Qd[:0], 5)
    assert ids.shape == (0, 5)


def test_sharded_build_and_merge(blsh, orc, c1):
    """Shard emulation on one GPU: world = 4 indexes over disjoint leaf ranges;
    their packed lists merged with blsh_merge_topk equal the unsharded result
    bit for bit (each query has one owning leaf)."""
    X, Q = c1
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    full = blsh.blsh_build(Xd, n_leaves=8, M=8, W=4.0, seed=5)
    fi, fd, fn = full.query(Qd, 10, probe=1, n_probes=16)
    lists, counts = [], []
    for r in range(4):
        sh = blsh.blsh_build(Xd, n_leaves=8, M=8, W=4.0, seed=5, rank=r, world=4)
        inf = sh.info()
        assert (inf.leaf_lo, inf.leaf_hi) == (2 * r, 2 * r + 2)
        pk, nc = sh.query_packed(Qd, 10, probe=1, n_probes=16)
        lists.append(pk)
        counts.append(nc)
    packed = torch.stack(lists).contiguous()
    mi, md = blsh.blsh_merge_topk(packed, 4, len(Q), 10)
    torch.cuda.synchronize()
    assert torch.equal(mi, fi) and torch.equal(md, fd)
    assert torch.equal(torch.stack(counts).sum(0), fn)
    # every query is owned by exactly one shard
    assert torch.all((torch.stack(counts) > 0).sum(0) <= 1)


@pytest.mark.parametrize("probe,T", [(0, 1), (1, 8)])
def test_sharded_hierarchy_global_median(blsh, orc, c1, probe, T):
    """Batch-median tau on a sharded index (R18): blsh_query_base_counts per
    shard, summed (what the SUM all-reduce of sharded.py does), passed as
    global_base -> merged result == the single-GPU result == the oracle's."""
    X, Q = c1
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    full = blsh.blsh_build(Xd, n_leaves=8, M=8, W=4.0, seed=5)
    fi, fd, fn = full.query(Qd, 10, probe=probe, n_probes=T, hierarchy=1)
    ox = orc.OracleIndex(X, G=8, M=8, W=4.0, seed=5)
    oi, od, onc = ox.query(Q, 10, probe=probe, T=T, hierarchy=1)
    assert np.array_equal(fn.cpu().numpy(), onc)
    shards = [blsh.blsh_build(Xd, n_leaves=8, M=8, W=4.0, seed=5, rank=r, world=2) for r in range(2)]
    with pytest.raises(blsh.BlshError):     # a sharded index cannot take the median of its own half
        shards[0].query_packed(Qd, 10, probe=probe, n_probes=T, hierarchy=1)
    gb = sum(s.base_counts(Qd, probe=probe, n_probes=T) for s in shards)
    assert np.array_equal(gb.cpu().numpy(), ox.get("q_base"))
    lists = [s.query_packed(Qd, 10, probe=probe, n_probes=T, hierarchy=1, global_base=gb)[0] for s in shards]
    mi, md = blsh.blsh_merge_topk(torch.stack(lists).contiguous(), 2, len(Q), 10)
    torch.cuda.synchronize()
    assert torch.equal(mi, fi) and torch.equal(md, fd)
    # host output of the base counts, and widening with an explicit tau ignores global_base
    hb = shards[1].base_counts(Q, probe=probe, n_probes=T)
    assert isinstance(hb, np.ndarray) and np.array_equal(hb, shards[1].base_counts(Qd, probe=probe, n_probes=T).cpu().numpy())


def test_merge_topk_against_numpy(blsh):
    rng = np.random.default_rng(9)
    L, nq, k = 5, 37, 13
    d2 = np.sort(rng.random((L, nq, k)).astype(np.float32), axis=2)
    ids = rng.integers(0, 2 ** 31, (L, nq, k)).astype(np.uint64)
    pk = (d2.view(np.uint32).astype(np.uint64) << np.uint64(32)) | ids
    pk[1, :, 5:] = np.uint64(0x7F800000FFFFFFFF)      # padding
    order = np.sort(pk.transpose(1, 0, 2).reshape(nq, -1), axis=1)
    order = np.where(order == np.uint64(0x7F800000FFFFFFFF), np.uint64(2 ** 64 - 1), order)
    order.sort(axis=1)
    t = torch.from_numpy(pk.view(np.int64)).cuda()
    mi, md = blsh.blsh_merge_topk(t, L, nq, k)
    mi, md = mi.cpu().numpy(), md.cpu().numpy()
    want = order[:, :k]
    assert np.array_equal(mi, (want & np.uint64(0xFFFFFFFF)).astype(np.int64))
    assert np.array_equal(md.view(np.uint32), (want >> np.uint64(32)).astype(np.uint32))


def test_c2_full(blsh, orc):
    """BASELINE configs[1] at full size: LabelMe-shaped 22k x 512, 1000 queries, k = 50."""
    cfg = synth.CONFIGS["c2"]
    X, Q = synth.make_dataset(cfg)
    if cfg.L == 1:
        ix, ox = build_pair(blsh, orc, X, G=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index)
        compare_build(ix, ox)
        run_query_pair(ix, ox, X, Q, cfg.k)
    else:   # standard LSH with L tables per subgroup (R24): the L-table parity helpers
        import test_gpu_tables as tt
        ix, ox = tt.build_pair(blsh, orc, X, cfg.L, G=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index)
        tt.run_pair(ix, ox, X, Q, cfg.k, cfg.L, probe=cfg.probe, T=cfg.T)


def test_warp_shortlist_fallback(blsh, orc, c1, monkeypatch):
    """The one-warp-per-(query, chunk) short-list (used when the tiled kernel's
    shared memory does not fit, e.g. d > 512) against the oracle."""
    X, Q = c1
    monkeypatch.setenv("BLSH_SHORTLIST", "warp")
    ix, ox = build_pair(blsh, orc, X, G=4, M=8, W=4.0, seed=11)
    run_query_pair(ix, ox, X, Q, 10, probe=1, T=16)
    run_query_pair(ix, ox, X, Q, 50, probe=1, T=4, hierarchy=1)
    assert ix.stats().tiled == 0
    monkeypatch.delenv("BLSH_SHORTLIST")
    run_query_pair(ix, ox, X, Q, 10, probe=1, T=16)
    ix.query(torch.from_numpy(Q).cuda(), 10, probe=1, n_probes=16)
    assert ix.stats().tiled == 0, "batches of <= 128 queries take the warp short-list by default"
    Q2 = np.concatenate([Q] * 11)                   # 1 100 queries (> 1 024): the tiled path
    run_query_pair(ix, ox, X, Q2, 10, probe=1, T=16)
    assert ix.stats().tiled >= 1


def test_large_d_uses_fallback(blsh, orc):
    mix = synth.mixture(1000, 8, 8, 0.2, 5)
    X = synth.sample_points(mix, 2500, 6)
    Q = synth.sample_points(mix, 30, 7)
    ix, ox = build_pair(blsh, orc, X, G=2, M=6, W=3.0)
    run_query_pair(ix, ox, X, Q, 10, probe=1, T=8)
    assert ix.stats().tiled == 0


@pytest.mark.parametrize("mode", ["simt", "tc"])
def test_tiled_shortlist_variants(blsh, orc, c1, monkeypatch, mode):
    """Both query-tiled short-list kernels (SIMT and the tensor-core screen with
    exact rescoring) against the oracle, k <= 16 so both are eligible."""
    X, Q = c1
    if mode == "simt":
        monkeypatch.setenv("BLSH_SHORTLIST", "simt")
    else:
        monkeypatch.setenv("BLSH_SHORTLIST", "tc")
    ix, ox = build_pair(blsh, orc, X, G=4, M=8, W=4.0, seed=21)
    for k, T in [(1, 1), (10, 16), (16, 64), (50, 16), (64, 8)] + ([(32, 16)] if mode == "tc" else []):
        run_query_pair(ix, ox, X, Q, k, probe=1 if T > 1 else 0, T=T)
        assert ix.stats().tiled == (1 if mode == "simt" else 2)


def _query_mode(ix, Q, k, mode, monkeypatch, **kw):
    monkeypatch.setenv("BLSH_SHORTLIST", mode)
    ids, d2, nc = ix.query(torch.from_numpy(Q).cuda(), k, **kw)
    torch.cuda.synchronize()
    tiled = ix.stats().tiled
    monkeypatch.delenv("BLSH_SHORTLIST")
    return ids.cpu().numpy(), d2.cpu().numpy(), nc.cpu().numpy(), tiled


@pytest.mark.parametrize("shape", ["lowrank384", "d512", "dup_overflow"])
def test_tc_screen_equals_warp(blsh, orc, monkeypatch, shape):
    """The tensor-core screen only decides which pairs get exact fp32 work, and its exact
    rescoring (k_tc_rescore, and the overflow path) uses the warp short-list's partial-sum
    order, so the two short-lists must agree bit for bit (ids and d^2 bits).  lowrank384:
    the C3/C4 shape (tight low-rank clusters far from the origin, where the screen's bound
    matters); d512: the largest d_stride the TC kernel takes; dup_overflow: 10 points
    repeated 1000x, so hundreds of pairs tie inside the screen margin and the per-warp
    pair buffers overflow."""
    if shape == "lowrank384":
        mix = synth.mixture(384, 64, 16, 0.02, 31)
        X = synth.sample_points(mix, 20000, 32)
        Q = synth.sample_points(mix, 400, 33)
        G, W, T = 4, 1.2, 16
    elif shape == "d512":
        mix = synth.mixture(512, 32, 16, 0.02, 41)
        X = synth.sample_points(mix, 12000, 42)
        Q = synth.sample_points(mix, 200, 43)
        G, W, T = 4, 1.6, 8
    else:
        mix = synth.mixture(128, 8, 8, 0.05, 51)
        base = synth.sample_points(mix, 10, 52)
        X = np.repeat(base, 1000, axis=0)
        Q = synth.sample_points(mix, 100, 53)
        G, W, T = 2, 3.0, 4
    ix, ox = build_pair(blsh, orc, X, G=G, M=8, W=W, seed=5)
    for k in (1, 10, 16, 17, 24, 32, 33, 50, 64):
        a = _query_mode(ix, Q, k, "warp", monkeypatch, probe=1, n_probes=T)
        b = _query_mode(ix, Q, k, "tc", monkeypatch, probe=1, n_probes=T)
        assert a[3] == 0 and b[3] == 2
        np.testing.assert_array_equal(a[2], b[2])
        np.testing.assert_array_equal(a[0], b[0])
        np.testing.assert_array_equal(a[1].view(np.uint32), b[1].view(np.uint32))
    run_query_pair(ix, ox, X, Q[:60], 10, probe=1, T=T)


def test_sharded_merge_against_oracle(blsh, orc):
    """SURVEY §8(e) against the oracle directly: world = 4 leaf shards (each answers its
    compacted ~1 250 owned queries on the tiled tcgen05 screen), packed lists merged with
    blsh_merge_topk; counts equal the oracle's |A(q)| and the merged top-k passes check_topk
    against the oracle's single-index answer."""
    X, Q = synth.make_dataset(synth.CONFIGS["c1"], n=10000, nq=5000)
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    ox = orc.OracleIndex(X, G=8, M=8, W=4.0, seed=5)
    oi, od, onc = ox.query(Q, 10, probe=1, T=16)
    lists, counts = [], []
    for r in range(4):
        sh = blsh.blsh_build(Xd, n_leaves=8, M=8, W=4.0, seed=5, rank=r, world=4)
        pk, nc = sh.query_packed(Qd, 10, probe=1, n_probes=16)
        lists.append(pk)
        counts.append(nc)
        sh.close()
    packed = torch.stack(lists).contiguous()
    mi, md = blsh.blsh_merge_topk(packed, 4, len(Q), 10)
    torch.cuda.synchronize()
    assert np.array_equal(torch.stack(counts).sum(0).cpu().numpy(), onc)
    check_topk(mi.cpu().numpy(), md.cpu().numpy(), oi, od, X, Q, cands=ox.candidates())
