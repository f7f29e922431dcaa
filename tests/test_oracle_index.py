"""Oracle pins: RP-tree, table, candidate sets (P:43, P:88,
P:132), short-list and brute force, Eq. 3."""
import math

import numpy as np
import pytest

import synth


@pytest.fixture(scope="module")
def c1():
    cfg = synth.CONFIGS["c1"]
    X, Q = synth.make_dataset(cfg)
    return X, Q


@pytest.fixture(scope="module")
def c1_index(orc, c1):
    X, _ = c1
    return orc.OracleIndex(X, G=4, M=8, W=4.0, seed=42)


def _np_knn(X, Q, k):
    d = ((Q.astype(np.float64)[:, None, :] - X.astype(np.float64)[None, :, :]) ** 2).sum(-1)
    ids = np.empty((Q.shape[0], k), np.int64)
    for i in range(Q.shape[0]):
        o = np.lexsort((np.arange(X.shape[0]), d[i]))[:k]
        ids[i] = o
    return ids, d


def test_bruteforce_vs_numpy(orc):
    rng = np.random.default_rng(0)
    X = rng.standard_normal((700, 13)).astype(np.float32)
    X[100] = X[5]                                     # exact duplicate -> tie by id
    Q = rng.standard_normal((30, 13)).astype(np.float32)
    Q[0] = X[5]
    for k in (1, 7, 50):
        ids, d2 = orc.bruteforce(X, Q, k)
        rid, dm = _np_knn(X, Q, k)
        assert np.array_equal(ids, rid)
        assert np.allclose(d2, np.take_along_axis(dm, rid, 1), rtol=1e-6)
    ids, d2 = orc.bruteforce(X[:3], Q[:2], 5)         # k > n: padding (R22)
    assert np.all(ids[:, 3:] == -1) and np.all(np.isinf(d2[:, 3:]))


def test_mean_rule_statistics(orc, c1, c1_index):
    X, _ = c1
    mu = c1_index.get("mu")
    da2 = c1_index.get("da2")
    m = X.astype(np.float64).mean(0)
    assert np.allclose(mu[0], m, rtol=0, atol=1e-6)
    ref = 2.0 * np.mean(((X.astype(np.float64) - mu[0].astype(np.float64)) ** 2).sum(1))
    assert math.isclose(da2[0], ref, rel_tol=1e-5)


def test_tree_balance_and_routing(orc, c1, c1_index):
    X, _ = c1
    leaf = c1_index.get("leaf")
    assert np.array_equal(np.bincount(leaf, minlength=4), [2500] * 4)       # median splits
    # route(x) == leaf(x): query the data points themselves
    c1_index.query(X[:2000], 1)
    assert np.array_equal(c1_index.get("q_leaf"), leaf[:2000])
    # hyperplane nodes: the median value is the split (<= goes left)
    ntype, theta, dirs = c1_index.get("ntype"), c1_index.get("theta"), c1_index.get("dirs")
    assert np.all(ntype == 0)
    s = X.astype(np.float64) @ dirs[0].astype(np.float64)
    assert abs(np.sort(s)[(len(s) - 1) // 2] - theta[0]) < 1e-4
    sc = np.array([orc.dot_canonical(dirs[0], x) for x in X], np.float32)
    assert np.sort(sc)[(len(sc) - 1) // 2] == theta[0]          # lower median (R5)
    assert np.sum(sc <= theta[0]) == 5000


def test_diameter_bounds(orc):
    """r_m <= Delta(S) <= min(sqrt(3) r_1, sqrt(5 - 2 sqrt(3)) r_m)."""
    rng = np.random.default_rng(1)
    worst = 0.0
    for trial in range(120):
        n = int(rng.integers(2, 60))
        d = int(rng.integers(1, 12))
        X = (rng.standard_normal((n, d)) * rng.uniform(0.1, 3, d)).astype(np.float32)
        est2, r12, sel = orc.diameter_estimate(X, np.arange(n), m=40)
        D = math.sqrt(max(((X[:, None, :].astype(np.float64) - X[None]) ** 2).sum(-1).max(), 0))
        rm = math.sqrt(est2)
        r1 = math.sqrt(r12)
        tol = 1e-5 * (D + 1e-12)
        assert rm <= D + tol
        assert D <= min(math.sqrt(3) * r1, math.sqrt(5 - 2 * math.sqrt(3)) * rm) + tol
        worst = max(worst, D / rm if rm > 0 else 1.0)
    assert worst <= math.sqrt(5 - 2 * math.sqrt(3)) + 1e-6


def test_sphere_split_with_outliers(orc):
    """Dense core + 0.5% far outliers: Delta^2 >> c * Delta_A^2 triggers the
    distance-from-mean split of RP-tree mean ([20])."""
    rng = np.random.default_rng(2)
    n, d = 4000, 24
    X = (0.1 * rng.standard_normal((n, d))).astype(np.float32)
    out = rng.choice(n, 20, replace=False)
    X[out] += (40.0 * rng.standard_normal((20, d))).astype(np.float32)
    ix = orc.OracleIndex(X, G=2, M=4, W=1.0, seed=3)
    assert ix.get("ntype")[0] == 1
    assert ix.get("diam2")[0] > 10.0 * ix.get("da2")[0]
    leaf = ix.get("leaf")
    assert abs(np.sum(leaf == 0) - np.sum(leaf == 1)) <= 1
    ix.query(X, 1)
    assert np.array_equal(ix.get("q_leaf"), leaf)
    # the far outliers are all on the far (right) side
    assert np.all(leaf[out] == 1)
    # max rule on the same data never uses the sphere split
    ix2 = orc.OracleIndex(X, G=2, M=4, W=1.0, seed=3, rp_rule=1)
    assert ix2.get("ntype")[0] == 0


def test_table_invariants(orc, c1_index):
    ix = c1_index
    n = ix.n
    perm, leaf, key = ix.get("perm"), ix.get("leaf"), ix.get("key")
    assert np.array_equal(np.sort(perm), np.arange(n))
    sk = [(int(leaf[i]), int(key[i, 0]), int(key[i, 1]), int(i)) for i in perm]
    assert sk == sorted(sk)
    ukey, uleaf, uoff = ix.get("ukey"), ix.get("uleaf"), ix.get("uoff")
    assert uoff[0] == 0 and uoff[-1] == n and np.all(np.diff(uoff) > 0)
    for u in range(ix.nu):
        ids = perm[uoff[u]:uoff[u + 1]]
        assert np.all(leaf[ids] == uleaf[u])
        assert np.all(key[ids, 0] == ukey[u, 0]) and np.all(key[ids, 1] == ukey[u, 1])
    for u in range(1, ix.nu):            # maximal runs: neighbours differ
        assert (uleaf[u], ukey[u, 0], ukey[u, 1]) != (uleaf[u - 1], ukey[u - 1, 0], ukey[u - 1, 1])
    # key is the Morton code of the stored code
    code = ix.get("code")
    for i in range(0, n, 997):
        assert orc.morton_encode(code[i]) == (int(key[i, 0]) << 64) | int(key[i, 1])


def _points_with_key(ix, g, k2):
    leaf, key = ix.get("leaf"), ix.get("key")
    return set(np.nonzero((leaf == g) & (key[:, 0] == k2[0]) & (key[:, 1] == k2[1]))[0].tolist())


def test_standard_candidates_are_the_home_bucket(orc, c1, c1_index):
    """A(v) = items with the same bi-level code (leaf, H(v))."""
    _, Q = c1
    ix = c1_index
    ids, d2, nc = ix.query(Q, 10)
    cands = ix.candidates()
    ql, qk, oor = ix.get("q_leaf"), ix.get("q_key"), ix.get("q_oor")
    for q in range(len(Q)):
        want = set() if oor[q] else _points_with_key(ix, ql[q], qk[q])
        assert set(cands[q].tolist()) == want and nc[q] == len(want)
        # query's own code: floor of its projections with its leaf's parameters
        t, h = orc.hash_point(ix.get("A")[ql[q]], ix.get("b")[ql[q]], 4.0, Q[q])
        assert np.array_equal(h, ix.get("q_code")[q])


def test_multiprobe_and_lattice_candidates(orc, c1):
    X, Q = c1
    Q = Q[:40]
    ix = orc.OracleIndex(X, G=4, M=8, W=4.0, seed=42)
    ix.query(Q, 10, probe=1, T=12)
    cands = ix.candidates()
    pk, pv, ql = ix.get("q_pkey"), ix.get("q_pvalid"), ix.get("q_leaf")
    t = ix.get("q_t")
    for q in range(len(Q)):
        deltas, _ = orc.multiprobe_deltas(t[q], 12)
        h = np.floor(t[q]).astype(np.int32)
        for p in range(12):
            code = h + (deltas[p - 1] if p else 0)
            assert orc.morton_encode(code) == (int(pk[q, p, 0]) << 64) | int(pk[q, p, 1])
        want = set()
        for p in range(12):
            if pv[q, p]:
                want |= _points_with_key(ix, ql[q], pk[q, p])
        assert set(cands[q].tolist()) == want
    e8 = orc.OracleIndex(X, G=4, M=8, W=4.0, seed=42, quantizer=1)
    e8.query(Q, 10, probe=2, T=20)
    cands = e8.candidates()
    pk, pv, ql = e8.get("q_pkey"), e8.get("q_pvalid"), e8.get("q_leaf")
    roots = orc.e8_roots()
    t, code = e8.get("q_t"), e8.get("q_code")
    for q in range(len(Q)):
        assert np.array_equal(code[q], orc.e8_decode(t[q]))
        order = orc.lattice_order(t[q], code[q], 20)
        for p in range(20):
            c = code[q] + (roots[order[p - 1]] if p else 0)
            assert orc.morton_encode(c) == (int(pk[q, p, 0]) << 64) | int(pk[q, p, 1])
        want = set()
        for p in range(20):
            if pv[q, p]:
                want |= _points_with_key(e8, ql[q], pk[q, p])
        assert set(cands[q].tolist()) == want


def test_all_buckets_probed_gives_exact_knn(orc):
    """G=1 and a hierarchy threshold of |S|: A(v) = S, so the short-list
    returns the exact k-NN (recall 1)."""
    rng = np.random.default_rng(4)
    X = rng.standard_normal((1500, 20)).astype(np.float32)
    Q = rng.standard_normal((25, 20)).astype(np.float32)
    ix = orc.OracleIndex(X, G=1, M=6, W=0.7, seed=9)
    ids, d2, nc = ix.query(Q, 15, hierarchy=1, min_cand=len(X))
    assert np.all(nc == len(X))
    bi, bd = orc.bruteforce(X, Q, 15)
    assert np.array_equal(ids, bi) and np.array_equal(d2, bd)


def test_hierarchy_widening_rules(orc, c1):
    X, Q = c1
    ix = orc.OracleIndex(X, G=4, M=8, W=4.0, seed=42)
    ids0, _, nc0 = ix.query(Q, 10)
    base = ix.get("q_base")
    assert np.array_equal(base, nc0)
    ids, _, nc = ix.query(Q, 10, hierarchy=1)            # tau = lower median
    tau = int(np.sort(nc0)[(len(nc0) - 1) // 2])
    assert ix.tau == tau
    lvl = ix.get("q_level")
    cand = ix.candidates()
    cand0 = None
    leaf, key = ix.get("leaf"), ix.get("key")
    ql, qcode = ix.get("q_leaf"), ix.get("q_code")
    for q in range(len(Q)):
        if nc0[q] >= tau:
            assert lvl[q] == 0 and nc[q] == nc0[q]
            continue
        assert lvl[q] % 8 == 0 and lvl[q] > 0
        assert nc[q] >= min(tau, np.sum(leaf == ql[q]))
        # candidates = points of the leaf whose Eq. 8 ancestor matches the query's
        anc = int(lvl[q]) // 8
        hk = orc.morton_encode(np.clip(qcode[q], -2**15, 2**15 - 1))
        inleaf = np.nonzero(leaf == ql[q])[0]
        kk = np.array([(int(key[i, 0]) << 64) | int(key[i, 1]) for i in inleaf], dtype=object)
        shift = anc * 8
        want = set(inleaf[[(int(v) >> shift) == (hk >> shift) for v in kk]].tolist())
        assert want.issubset(set(cand[q].tolist()))
        # one level less would not have reached tau (first sufficient level)
        if anc > 1:
            prev = sum((int(v) >> ((anc - 1) * 8)) == (hk >> ((anc - 1) * 8)) for v in kk)
            assert prev < tau
    # explicit tau larger than any leaf -> whole leaf
    ix.query(Q[:10], 10, hierarchy=1, min_cand=10 ** 9)
    ql = ix.get("q_leaf")
    _, _, ncw = ix.query(Q[:10], 10, hierarchy=1, min_cand=10 ** 9)
    assert np.array_equal(ncw, np.bincount(leaf, minlength=4)[ql])


def test_recall_eq3_invariant(orc, c1):
    """Eq. 3: |N ∩ I| = |N ∩ A| when I is the top-k of A."""
    X, Q = c1
    ix = orc.OracleIndex(X, G=4, M=8, W=4.0, seed=42)
    ids, d2, nc = ix.query(Q, 10, probe=1, T=8)
    cand = ix.candidates()
    gi, gd = orc.bruteforce(X, Q, 10)
    for q in range(len(Q)):
        N = set(gi[q].tolist())
        assert len(N & set(ids[q].tolist())) == len(N & set(cand[q].tolist()))


def test_shortlist_is_sorted_topk_of_candidates(orc, c1):
    X, Q = c1
    ix = orc.OracleIndex(X, G=4, M=8, W=4.0, seed=42)
    ids, d2, nc = ix.query(Q, 50, probe=1, T=4)
    cand = ix.candidates()
    for q in range(len(Q)):
        c = cand[q]
        dd = ((X[c].astype(np.float64) - Q[q].astype(np.float64)) ** 2).sum(1)
        o = np.lexsort((c, dd))[:50]
        m = min(50, len(c))
        assert np.array_equal(ids[q, :m], c[o][:m])
        assert np.all(ids[q, m:] == -1) and np.all(np.isinf(d2[q, m:]))
        assert np.array_equal(d2[q, :m], dd[o][:m].astype(np.float32))


def test_invalid_arguments(orc, c1):
    X, Q = c1
    with pytest.raises(orc.OracleError):
        orc.OracleIndex(X, G=3)
    with pytest.raises(orc.OracleError):
        orc.OracleIndex(X, G=4, M=7, quantizer=1)
    ix = orc.OracleIndex(X[:500], G=2, M=8, W=4.0)
    with pytest.raises(orc.OracleError):
        ix.query(Q, 10, probe=2, T=4)                   # lattice needs an E8 index
    with pytest.raises(orc.OracleError):
        ix.query(Q, 0)
    # W so small that codes leave the 16-bit Morton range (R9)
    with pytest.raises(orc.OracleError) as e:
        orc.OracleIndex(X[:500] * 1e4, G=2, M=8, W=1e-3)
    assert e.value.args[1] == 4


@pytest.mark.parametrize("probe,T,hier", [(1, 16, 0), (0, 1, 1), (3, 4, 0)])
def test_nonfinite_queries_have_no_candidates(orc, c1, c1_index, probe, T, hier):
    """R30: a query whose projection is non-finite has no probes and no candidates;
    the rest of the batch is answered exactly as without it (min_cand fixed, so the
    batch median does not move)."""
    X, Q = c1
    Qb = Q.copy()
    Qb[2, 0] = np.nan
    Qb[5, 3] = np.inf
    ids_b, d2_b, nc_b = c1_index.query(Qb, 10, probe=probe, T=T, hierarchy=hier, min_cand=50)
    oor = c1_index.get("q_oor")
    assert oor[2] == 5 and oor[5] == 5
    assert nc_b[2] == 0 and nc_b[5] == 0
    assert np.all(ids_b[[2, 5]] == -1) and np.all(np.isinf(d2_b[[2, 5]]))
    assert not np.any(c1_index.get("q_pvalid").reshape(len(Q), T)[[2, 5]])
    ids, d2, nc = c1_index.query(Q, 10, probe=probe, T=T, hierarchy=hier, min_cand=50)
    good = [q for q in range(len(Q)) if q not in (2, 5)]
    assert np.array_equal(ids[good], ids_b[good]) and np.array_equal(nc[good], nc_b[good])


def test_max_rule_jitter_closed_form(orc):
    """R4 max rule with jitter ([20]): theta_j - theta_0 = (2u - 1) j |x0 - y| / sqrt(d),
    u = U(seed, stream (4, 0, v), 0) (R2, pinned by the SplitMix64 known answers), x0 the
    node's lowest-id member, y its farthest member from x0 (ties -> lowest id).  The node
    membership and |x0 - y| are recomputed here in numpy fp64; a sign, index or scale error
    in the oracle's jitter branch moves theta by far more than the fp32 tolerance."""
    rng = np.random.default_rng(11)
    n, d, j, seed = 3000, 24, 0.25, 77   # [20]'s j = 6 empties one child at this size
    X = rng.standard_normal((n, d)).astype(np.float32)
    o0 = orc.OracleIndex(X, G=4, M=4, W=1.0, seed=seed, rp_rule=1, rp_max_jitter=0.0)
    oj = orc.OracleIndex(X, G=4, M=4, W=1.0, seed=seed, rp_rule=1, rp_max_jitter=j)
    dirs = oj.get("dirs").astype(np.float64)
    assert np.array_equal(o0.get("dirs"), oj.get("dirs"))
    th0, thj = o0.get("theta"), oj.get("theta")
    leaf = oj.get("leaf")
    members = {0: np.arange(n), 1: np.nonzero(leaf < 2)[0], 2: np.nonzero(leaf >= 2)[0]}
    X64 = X.astype(np.float64)
    shifts = []
    for v, S in members.items():
        x0 = X64[S[0]]
        dist2 = ((X64[S] - x0) ** 2).sum(1)
        y = S[int(np.argmax(dist2))]
        u = orc.rng_uniform(seed, (4 << 24) + v, 0)
        delta = (2.0 * u - 1.0) * j * math.sqrt(dist2.max()) / math.sqrt(d)
        # the jitter-free median of the SAME node (node v's members under the jittered tree)
        s = np.sort(np.array([np.float32(np.dot(dirs[v], X64[i])) for i in S]))
        med = float(s[(len(S) - 1) // 2])
        if v == 0:
            assert float(th0[0]) == pytest.approx(med, rel=1e-5, abs=1e-5)
            assert float(thj[0]) - float(th0[0]) == pytest.approx(delta, rel=1e-4, abs=4e-6)
        else:
            assert float(thj[v]) - med == pytest.approx(delta, rel=1e-4, abs=5e-5)
        shifts.append(delta)
    assert len(set(np.round(shifts, 9))) == 3, "each node draws its own u"
    # balance moves by exactly the points between the two thetas at the root
    s_root = X64 @ dirs[0]
    lo, hi = sorted([float(th0[0]), float(thj[0])])
    moved = np.count_nonzero((s_root > lo) & (s_root <= hi))
    assert abs(np.count_nonzero(leaf < 2) - np.count_nonzero(o0.get("leaf") < 2)) == moved
