"""GPU parity for the large-k short-list (64 < k <= 1024; the paper evaluates
k = 500): every candidate's packed (d^2, id) key is emitted and a
per-query block radix select keeps the k smallest (shortlist.cu, k_select).

Same bar as the k <= 64 path: candidate sets bit-exact, distances within
1e-5 relative of the oracle's fp64 distances, ids equal except ties.
"""
import numpy as np
import pytest

import synth
from parity_utils import check_topk
from test_gpu_parity import build_pair, run_query_pair

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def blsh():
    if not torch.cuda.is_available():
        pytest.skip("needs CUDA")
    from paper_conf_icde_panm12_b200 import blsh as b
    b.lib()
    return b


@pytest.fixture(scope="module")
def c1():
    return synth.make_dataset(synth.CONFIGS["c1"])


@pytest.fixture(scope="module")
def c1_pair(blsh, orc, c1):
    X, _ = c1
    return build_pair(blsh, orc, X, G=4, M=8, W=4.0, seed=42)


@pytest.mark.parametrize("k", [65, 100, 500, 1024])
def test_large_k_standard(c1_pair, c1, k):
    """Standard probing: many buckets hold fewer than k points (padding), some more."""
    X, Q = c1
    run_query_pair(*c1_pair, X, Q, k)


@pytest.mark.parametrize("k,T", [(500, 64), (200, 16)])
def test_large_k_multiprobe(c1_pair, c1, k, T):
    X, Q = c1
    run_query_pair(*c1_pair, X, Q, k, probe=1, T=T)


def test_large_k_hierarchy(c1_pair, c1):
    """Widened candidate sets (thousands of rows) exercise all radix-select passes."""
    X, Q = c1
    run_query_pair(*c1_pair, X, Q, 1024, probe=1, T=4, hierarchy=1, min_cand=2000)


def test_large_k_prefix_equals_small_k(c1_pair, c1, monkeypatch):
    """The k smallest keys are unique, so the first 64 of a k = 700 list are the
    warp short-list's k = 64 list bit for bit (same distance arithmetic, R22;
    register top-k vs emit + radix select)."""
    ix, _ = c1_pair
    _, Q = c1
    Qd = torch.from_numpy(Q).cuda()
    monkeypatch.setenv("BLSH_SHORTLIST", "warp")
    i64, d64, n64 = ix.query(Qd, 64, probe=1, n_probes=32)
    monkeypatch.delenv("BLSH_SHORTLIST")
    i7, d7, n7 = ix.query(Qd, 700, probe=1, n_probes=32)
    torch.cuda.synchronize()
    assert torch.equal(i64, i7[:, :64]) and torch.equal(d64.view(torch.int32), d7[:, :64].contiguous().view(torch.int32))
    assert torch.equal(n64, n7)


def test_large_k_duplicate_rows(blsh, orc):
    """Many identical rows: equal d^2, distinct ids -> ties broken by id, exactly."""
    rng = np.random.default_rng(5)
    base = rng.standard_normal((300, 24)).astype(np.float32)
    X = np.repeat(base, 10, axis=0)
    rng.shuffle(X)
    Q = (X[rng.choice(len(X), 40, replace=False)] + 0.01 * rng.standard_normal((40, 24))).astype(np.float32)
    ix, ox = build_pair(blsh, orc, X, G=2, M=4, W=8.0, seed=3)
    ids, d2, nc = run_query_pair(ix, ox, X, Q, 300, probe=1, T=9)
    oi, od, _ = ox.query(Q, 300, probe=1, T=9)
    # ties are exact duplicates of one row: the (d^2, id) order is total, so ids match exactly
    fin = np.isfinite(od)
    assert np.array_equal(ids[fin], oi[fin])


def test_large_k_merge_topk_against_numpy(blsh):
    rng = np.random.default_rng(11)
    L, nq, k = 3, 29, 300
    d2 = np.sort(rng.random((L, nq, k)).astype(np.float32), axis=2)
    ids = rng.permutation(2 ** 20)[: L * nq * k].reshape(L, nq, k).astype(np.uint64)
    pk = (d2.view(np.uint32).astype(np.uint64) << np.uint64(32)) | ids
    pk.sort(axis=2)
    pk[1, :, 120:] = np.uint64(0x7F800000FFFFFFFF)      # a short rank
    pk[2, 3:6, :] = np.uint64(0x7F800000FFFFFFFF)        # a rank owning nothing for some queries
    allk = pk.transpose(1, 0, 2).reshape(nq, -1)
    allk = np.where(allk == np.uint64(0x7F800000FFFFFFFF), np.uint64(2 ** 64 - 1), allk)
    allk.sort(axis=1)
    t = torch.from_numpy(pk.view(np.int64)).cuda()
    mi, md = blsh.blsh_merge_topk(t, L, nq, k)
    mi, md = mi.cpu().numpy(), md.cpu().numpy()
    want = allk[:, :k]
    assert np.array_equal(mi, (want & np.uint64(0xFFFFFFFF)).astype(np.int64))
    assert np.array_equal(md.view(np.uint32), (want >> np.uint64(32)).astype(np.uint32))


def test_large_k_merge_short_lists(blsh):
    """Fewer real entries than k over all lists -> padded output (-1, +inf)."""
    L, nq, k = 2, 4, 100
    pk = np.full((L, nq, k), np.uint64(0x7F800000FFFFFFFF), np.uint64)
    for q in range(nq):
        for l in range(L):
            m = 10 * (q + l)
            d = np.sort(np.random.default_rng(q * 7 + l).random(m).astype(np.float32))
            ids = np.uint64(100000 * l + 1000 * q) + np.arange(m, dtype=np.uint64)
            pk[l, q, :m] = (d.view(np.uint32).astype(np.uint64) << np.uint64(32)) | ids
    t = torch.from_numpy(pk.view(np.int64)).cuda()
    mi, md = blsh.blsh_merge_topk(t, L, nq, k)
    mi, md = mi.cpu().numpy(), md.cpu().numpy()
    for q in range(nq):
        real = np.sort(np.concatenate([pk[l, q][pk[l, q] != np.uint64(0x7F800000FFFFFFFF)] for l in range(L)]))
        m = len(real)
        assert np.array_equal(mi[q, :m], (real & np.uint64(0xFFFFFFFF)).astype(np.int64))
        assert np.all(mi[q, m:] == -1) and np.all(np.isinf(md[q, m:]))


def test_large_k_unsupported(blsh, c1_pair, c1):
    ix, _ = c1_pair
    _, Q = c1
    with pytest.raises(Exception):
        ix.query(torch.from_numpy(Q).cuda(), 1025)


def test_large_k_sharded_merge_matches_single(blsh, orc, c1):
    """a6 with k = 256: two leaf shards + merge == the single-GPU list."""
    X, Q = c1
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    full = blsh.blsh_build(Xd, n_leaves=4, M=8, W=4.0, seed=42)
    i1, d1, _ = full.query(Qd, 256, probe=1, n_probes=8)
    parts = []
    for r in range(2):
        sh = blsh.blsh_build(Xd, n_leaves=4, M=8, W=4.0, seed=42, rank=r, world=2)
        pk, _ = sh.query_packed(Qd, 256, probe=1, n_probes=8)
        parts.append(pk)
    mi, md = blsh.blsh_merge_topk(torch.cat(parts).contiguous(), 2, len(Q), 256)
    torch.cuda.synchronize()
    assert torch.equal(mi, i1) and torch.equal(md.view(torch.int32), d1.view(torch.int32))


# Large k on the tensor-core path (64 < k <= 512): the fp16 screen keeps ceil(k/8) bounds per
# epilogue warp, every survivor gets the exact fp32 distance, k_select keeps the k smallest.
@pytest.mark.parametrize("k,T", [(65, 8), (100, 16), (500, 64), (512, 4)])
def test_large_k_tc_vs_oracle(c1_pair, c1, monkeypatch, k, T):
    X, Q = c1
    monkeypatch.setenv("BLSH_SHORTLIST", "tc")
    run_query_pair(*c1_pair, X, Q, k, probe=1, T=T)
    assert c1_pair[0].stats().tiled == 2


def test_large_k_tc_hierarchy_and_default_batch(c1_pair, c1):
    X, Q = c1
    Q3 = np.concatenate([Q] * 11)                   # 1 100 queries (> 1 024): the tiled path by default
    run_query_pair(*c1_pair, X, Q3, 300, probe=1, T=8, hierarchy=1)
    assert c1_pair[0].stats().tiled == 2


def _mode(ix, Q, k, mode, monkeypatch, **kw):
    monkeypatch.setenv("BLSH_SHORTLIST", mode)
    ids, d2, nc = ix.query(torch.from_numpy(Q).cuda(), k, **kw)
    torch.cuda.synchronize()
    t = ix.stats().tiled
    monkeypatch.delenv("BLSH_SHORTLIST")
    return ids.cpu().numpy(), d2.cpu().numpy(), nc.cpu().numpy(), t


@pytest.mark.parametrize("shape", ["lowrank384", "dup_overflow"])
def test_large_k_tc_equals_warp(blsh, orc, monkeypatch, shape):
    """Bit identity of the large-k TC path with the warp large-k path (ids, d^2 bits, counts);
    dup_overflow: 10 points repeated 1000x, so the per-warp pair buffers overflow and the
    items' rows are scored exhaustively."""
    if shape == "lowrank384":
        mix = synth.mixture(384, 64, 16, 0.02, 31)
        X = synth.sample_points(mix, 20000, 32)
        Q = synth.sample_points(mix, 400, 33)
        G, W, T = 4, 1.2, 16
    else:
        mix = synth.mixture(128, 8, 8, 0.05, 51)
        X = np.repeat(synth.sample_points(mix, 10, 52), 1000, axis=0)
        Q = synth.sample_points(mix, 100, 53)
        G, W, T = 2, 3.0, 4
    ix, ox = build_pair(blsh, orc, X, G=G, M=8, W=W, seed=5)
    for k in (65, 128, 500, 512):
        a = _mode(ix, Q, k, "warp", monkeypatch, probe=1, n_probes=T)
        b = _mode(ix, Q, k, "tc", monkeypatch, probe=1, n_probes=T)
        assert a[3] == 0 and b[3] == 2
        np.testing.assert_array_equal(a[2], b[2])
        np.testing.assert_array_equal(a[0], b[0])
        np.testing.assert_array_equal(a[1].view(np.uint32), b[1].view(np.uint32))
    monkeypatch.setenv("BLSH_SHORTLIST", "tc")
    run_query_pair(ix, ox, X, Q[:60], 200, probe=1, T=T)


def test_k_above_512_stays_on_warp_path(c1_pair, c1):
    X, Q = c1
    Q3 = np.concatenate([Q, Q, Q])
    run_query_pair(*c1_pair, X, Q3, 600, probe=1, T=4)
    assert c1_pair[0].stats().tiled == 0
