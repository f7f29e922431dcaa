"""Oracle pins for L > 1 hash tables ("L hash tables are used and each of
them is constructed independently with different dim-M hash functions";
A(v) = the points of the buckets the query's codes hit; P:241 the L-table
collision probability 1 - prod_i min(|a_i.u - a_i.v|, W) / W).  Readings R2,
R24 in DESIGN.md."""
import math

import numpy as np
import pytest
from scipy import stats

import synth


@pytest.fixture(scope="module")
def c1():
    X, Q = synth.make_dataset(synth.CONFIGS["c1"])
    return X, Q[:40]


def test_table_params_streams(orc):
    """Table 0 is the single-table draw; tables l > 0 are new independent
    N(0,1) / U[0,W) draws (KS tests), not copies or shifts of table 0."""
    A0, b0, _, _ = orc.gen_params(7, 4, 8, 64, 2.5)
    T0A, T0b = orc.gen_table_params(7, 0, 4, 8, 64, 2.5)
    assert np.array_equal(A0, T0A) and np.array_equal(b0, T0b)
    seen = [A0.ravel()]
    for l in (1, 2, 5):
        A, b = orc.gen_table_params(7, l, 4, 8, 64, 2.5)
        assert stats.kstest(A.ravel().astype(np.float64), "norm").pvalue > 1e-3
        assert np.all((b >= 0) & (b < 2.5))
        assert stats.kstest(b.ravel() / 2.5, "uniform").pvalue > 1e-3
        for s in seen:
            assert abs(np.corrcoef(s, A.ravel())[0, 1]) < 0.05
        seen.append(A.ravel())


def test_tables_share_the_tree(orc, c1):
    X, _ = c1
    ix = orc.OracleIndex(X, G=4, M=8, W=4.0, seed=42, L=3)
    for l in (1, 2):
        for what in ("dirs", "theta", "ntype", "mu", "leaf"):
            assert np.array_equal(ix.get(what, l), ix.get(what, 0)), what
        assert not np.array_equal(ix.get("A", l), ix.get("A", 0))
        # every table is a valid sorted table over the same leaves
        perm, leaf = ix.get("perm", l), ix.get("leaf", l)
        assert np.array_equal(np.sort(perm), np.arange(len(X)))
        assert np.all(np.diff(leaf[perm]) >= 0)


def _points_with_key(ix, l, g, k2):
    leaf, key = ix.get("leaf", l), ix.get("key", l)
    return set(np.nonzero((leaf == g) & (key[:, 0] == k2[0]) & (key[:, 1] == k2[1]))[0].tolist())


@pytest.mark.parametrize("probe,T", [(0, 1), (1, 6)])
def test_union_candidates_bruteforce(orc, c1, probe, T):
    """A(q) = union over tables of the points whose table-l key equals one of
    the query's valid table-l probe keys (brute-force scan of all points);
    each table's probe keys are the Morton keys of that table's own codes."""
    X, Q = c1
    L = 3
    ix = orc.OracleIndex(X, G=4, M=8, W=4.0, seed=42, L=L)
    ids, d2, nc = ix.query(Q, 10, probe=probe, T=T)
    cands = ix.candidates()
    per = [ix.candidates(table=l) for l in range(L)]
    for l in range(L):
        pk, pv, ql, t = ix.get("q_pkey", l), ix.get("q_pvalid", l), ix.get("q_leaf", l), ix.get("q_t", l)
        A, b, W = ix.get("A", l), ix.get("b", l), ix.get("W", l)
        for q in range(len(Q)):
            g = ql[q]
            t_ref, h = orc.hash_point(A[g], b[g], W[g], Q[q])
            assert np.array_equal(t_ref.view(np.uint32), t[q].view(np.uint32))
            assert orc.morton_encode(h) == (int(pk[q, 0, 0]) << 64) | int(pk[q, 0, 1])
            want = set()
            for p in range(T):
                if pv[q, p]:
                    want |= _points_with_key(ix, l, g, pk[q, p])
            assert set(per[l][q].tolist()) == want
    for q in range(len(Q)):
        u = set()
        for l in range(L):
            u |= set(per[l][q].tolist())
        assert set(cands[q].tolist()) == u
        assert nc[q] == len(u)
        # short-list over the union: the exact top-k of A(q) by (d2, id)
        cq = np.array(sorted(u), np.int64)
        if len(cq):
            dd = ((X[cq].astype(np.float64) - Q[q].astype(np.float64)) ** 2).sum(1)
            o = np.lexsort((cq, dd))[:10]
            m = len(o)
            assert np.array_equal(ids[q, :m], cq[o])
            assert np.array_equal(d2[q, :m], dd[o].astype(np.float32))
        assert np.all(ids[q, len(cq):] == -1)


def test_single_table_union_is_the_plain_query(orc, c1):
    X, Q = c1
    a = orc.OracleIndex(X, G=4, M=8, W=4.0, seed=42, L=1)
    i1, d1, n1 = a.query(Q, 10, probe=1, T=8)
    import ctypes as C
    lib = orc.lib()
    arr = (C.c_void_p * 1)(a._h)
    i2, d2, n2 = np.empty_like(i1), np.empty_like(d1), np.empty_like(n1)
    rc = lib.orc_query_union(arr, 1, orc._p(np.ascontiguousarray(Q)), len(Q), 10, 1, 8, orc._p(i2), orc._p(d2),
                             orc._p(n2))
    assert rc == 0
    assert np.array_equal(i1, i2) and np.array_equal(d1, d2) and np.array_equal(n1, n2)


def test_more_tables_more_recall(orc, c1):
    """Union semantics: A_L(q) grows with L, so recall (Eq. 3) never drops."""
    X, Q = c1
    gt, _ = orc.bruteforce(X, Q, 10)
    prev = None
    for L in (1, 2, 4):
        ix = orc.OracleIndex(X, G=4, M=8, W=2.0, seed=42, L=L)
        ix.query(Q, 10)
        c = ix.candidates()
        rec = np.mean([len(set(gt[q]) & set(c[q].tolist())) / 10 for q in range(len(Q))])
        if prev is not None:
            for q in range(len(Q)):
                assert set(prev[1][q].tolist()) <= set(c[q].tolist())
            assert rec >= prev[0]
        prev = (rec, c)


def test_L_table_collision_probability(orc):
    """with L tables of 1-D hashes, P[u, v share a bucket in >= 1 table]
    = 1 - prod_i min(|a_i.u - a_i.v|, W) / W (b_i ~ U[0,W) independent per
    table).  Over seeds, the empirical collision rate of the oracle's union
    candidate set matches the mean of the closed form."""
    rng = np.random.default_rng(8)
    d, W, L = 16, 1.0, 3
    u = rng.standard_normal(d).astype(np.float32)
    v = (u + 0.08 * rng.standard_normal(d)).astype(np.float32)
    X = np.stack([u, v])
    hits, expect = 0, 0.0
    trials = 500
    for seed in range(trials):
        ix = orc.OracleIndex(X, G=1, M=1, W=W, seed=1000 + seed, L=L)
        ix.query(u[None, :], 2)
        hits += int(1 in set(ix.candidates()[0].tolist()))
        miss = 1.0
        for l in range(L):
            a = ix.get("A", l)[0, 0].astype(np.float64)
            miss *= min(abs(float(a @ (u.astype(np.float64) - v.astype(np.float64)))), W) / W
        expect += 1.0 - miss
    p = expect / trials
    se = math.sqrt(max(p * (1 - p), 1e-3) / trials)
    assert abs(hits / trials - p) < 5 * se


def test_hierarchy_rejected_with_tables(orc, c1):
    X, Q = c1
    ix = orc.OracleIndex(X, G=4, M=8, W=4.0, seed=42, L=2)
    with pytest.raises(orc.OracleError):
        ix.query(Q, 10, hierarchy=1)
