"""Oracle pins for the E8 code hierarchy (Eq. 10; reading R27):
parent(c) = DECODE(c / 2) in lattice units (doubled codes: DECODE(c2 / 4));
P:162 scaling property (the parent of 2p is p for every lattice point p);
the parent is a nearest lattice point of c / 2 (Voronoi test against the 240
roots); the widening rule of P:171 + P:249 on an E8 index."""
import numpy as np
import pytest

import synth


def _random_e8(rng, n, scale=6):
    """Random E8 points in doubled coordinates (D8 or D8 + 1/2)."""
    out = []
    while len(out) < n:
        z = rng.integers(-scale, scale + 1, 8)
        if rng.random() < 0.5:
            if z.sum() % 2:
                z[0] += 1
            out.append(2 * z)
        else:
            h = 2 * z + 1                      # odd doubled coordinates = half-integers
            if (h.sum() // 2) % 2:             # sum of the half-integer coordinates must be even
                h[0] += 2
            out.append(h)
    return np.array(out, np.int32)


def _is_e8(c2):
    c2 = np.asarray(c2)
    if np.all(c2 % 2 == 0):
        return (c2 // 2).sum() % 2 == 0
    if np.all(c2 % 2 != 0):
        return (c2.sum() // 2) % 2 == 0
    return False


def test_scaling_property(orc):
    """the integer scaling of E8 is E8, so the parent of the code of 2p is p."""
    rng = np.random.default_rng(1)
    for c in _random_e8(rng, 300):
        assert _is_e8(c)
        assert np.array_equal(orc.e8_parent(2 * c), c)


def test_parent_is_nearest(orc):
    rng = np.random.default_rng(2)
    roots = orc.e8_roots().astype(np.float64) / 2.0
    for c in _random_e8(rng, 300, scale=40):
        par = orc.e8_parent(c)
        assert _is_e8(par)
        y = c.astype(np.float64) / 4.0        # half of the lattice point c / 2
        x = par.astype(np.float64) / 2.0
        d0 = ((y - x) ** 2).sum()
        d = ((y[None, :] - x[None, :] - roots) ** 2).sum(1)
        assert d0 <= d.min() + 1e-12
        # chains shrink to the origin's neighbourhood: |parent| <= |c| / 2 + covering radius
        assert np.sqrt((x ** 2).sum()) <= np.sqrt(((c / 2.0) ** 2).sum()) / 2 + 1.0 + 1e-9


def _chain(orc, c, j):
    for _ in range(j):
        c = orc.e8_parent(c)
    return c


@pytest.mark.parametrize("tau", [0, 400, 2000])
def test_e8_hierarchy_widening_rule(orc, tau):
    X, Q = synth.make_dataset(synth.CONFIGS["c1"])
    Q = Q[:30]
    ix = orc.OracleIndex(X, G=4, M=8, W=2.0, seed=42, quantizer=1)
    ix.query(Q, 10, probe=2, T=4, hierarchy=1, min_cand=tau)
    tau_used = ix.tau
    base, lvl, ql, code = ix.get("q_base"), ix.get("q_level"), ix.get("q_leaf"), ix.get("q_code")
    uleaf, uoff, perm, pcode = ix.get("uleaf"), ix.get("uoff"), ix.get("perm"), ix.get("code")
    cands = ix.candidates()
    full = orc.OracleIndex(X, G=4, M=8, W=2.0, seed=42, quantizer=1)
    full.query(Q, 10, probe=2, T=4)
    a0 = full.candidates()
    for q in range(len(Q)):
        if base[q] >= tau_used:
            assert lvl[q] == 0 and np.array_equal(cands[q], a0[q])
            continue
        bks = np.nonzero(uleaf == ql[q])[0]
        bcode = [pcode[perm[uoff[u]]] for u in bks]
        if lvl[q] > 32:                      # whole leaf
            want = set(np.nonzero(ix.get("leaf") == ql[q])[0].tolist())
        else:
            L = int(lvl[q])
            cq = _chain(orc, code[q], L)
            node = [u for u, c in zip(bks, bcode) if np.array_equal(_chain(orc, c, L), cq)]
            rows = sum(int(uoff[u + 1] - uoff[u]) for u in node)
            assert node and rows >= tau_used
            if L > 0:                        # the level below is not enough (no match or too small)
                cq1 = _chain(orc, code[q], L - 1)
                node1 = [u for u, c in zip(bks, bcode) if np.array_equal(_chain(orc, c, L - 1), cq1)]
                assert set(node1) <= set(node)
                assert sum(int(uoff[u + 1] - uoff[u]) for u in node1) < tau_used
            want = set()
            for u in node:
                want |= set(perm[uoff[u]:uoff[u + 1]].tolist())
        want |= set(a0[q].tolist())
        assert set(cands[q].tolist()) == want


def test_second_ring_is_the_e8_shells(orc):
    """Recursive probing (R26): the neighbours of the 240 neighbours are
    exactly the E8 vectors of norm^2 4 and 6 (theta series: 2160 and 6720, every
    one of them) and the 240 vectors 2r of norm^2 8."""
    s2 = orc.e8_second_ring()
    roots = orc.e8_roots()
    n2 = (s2.astype(np.int64) ** 2).sum(1)          # doubled coordinates: 4x the norm^2
    assert (n2 == 16).sum() == 2160 and (n2 == 24).sum() == 6720 and (n2 == 32).sum() == 240
    assert len({tuple(v) for v in s2}) == 9120
    assert all(_is_e8(v) for v in s2[::7])
    assert {tuple(v) for v in s2[n2 == 32]} == {tuple(2 * r) for r in roots}
    # canonical order: by norm, then lexicographic
    keys = [(int(n), tuple(int(x) for x in v)) for n, v in zip(n2, s2)]
    assert keys == sorted(keys)


def test_recursive_lattice_order(orc):
    rng = np.random.default_rng(4)
    s2 = orc.e8_second_ring().astype(np.float64) / 2.0
    for _ in range(20):
        y = (rng.standard_normal(8) * 3).astype(np.float32)
        c = orc.e8_decode(y)
        o241 = orc.lattice_order(y, c, 241)
        o256 = orc.lattice_order(y, c, 256)
        assert np.array_equal(o256[:240], o241)                  # the first ring first, unchanged
        ring = o256[240:] - 240
        assert np.all(ring >= 0)
        d = ((y.astype(np.float64) - c / 2.0 - s2) ** 2).sum(1)
        want = np.lexsort((np.arange(9120), d))[:15]
        assert np.array_equal(ring, want)


def _leaf_points_with_key(ix, g, k2):
    leaf, key = ix.get("leaf"), ix.get("key")
    return set(np.nonzero((leaf == g) & (key[:, 0] == k2[0]) & (key[:, 1] == k2[1]))[0].tolist())


def test_two_block_e8_hash_and_probes(orc):
    """M = 16 (ceil(M/8) E8 lattices, R28): the code is the two blocks'
    DECODEs; lattice probes move one block by one root, ordered by the fp64
    distance over all 16 coordinates (brute force over the 480 candidates)."""
    rng = np.random.default_rng(6)
    X = (rng.standard_normal((3000, 24)) * 0.5).astype(np.float32)
    Q = (X[:25] + 0.05 * rng.standard_normal((25, 24))).astype(np.float32)
    ix = orc.OracleIndex(X, G=2, M=16, W=1.0, seed=3, quantizer=1)
    assert ix.B == 8
    T = 40
    ix.query(Q, 10, probe=2, T=T)
    t, code, pk, pv, ql = ix.get("q_t"), ix.get("q_code"), ix.get("q_pkey"), ix.get("q_pvalid"), ix.get("q_leaf")
    roots = orc.e8_roots()
    cands = ix.candidates()
    for q in range(len(Q)):
        c = np.concatenate([orc.e8_decode(t[q, :8]), orc.e8_decode(t[q, 8:])])
        assert np.array_equal(code[q], c) and _is_e8(c[:8]) and _is_e8(c[8:])
        cand = []
        for x in range(480):
            p = c.copy()
            p[8 * (x // 240):8 * (x // 240) + 8] += roots[x % 240]
            cand.append(p)
        cand = np.array(cand)
        d = ((t[q].astype(np.float64)[None, :] - cand / 2.0) ** 2).sum(1)
        order = np.lexsort((np.arange(480), d))[:T - 1]
        want = set(_leaf_points_with_key(ix, ql[q], pk[q, 0]))
        for p in range(1, T):
            assert orc.morton_encode(cand[order[p - 1]]) == (int(pk[q, p, 0]) << 64) | int(pk[q, p, 1])
            if pv[q, p]:
                want |= _leaf_points_with_key(ix, ql[q], pk[q, p])
        assert set(cands[q].tolist()) == want


def test_two_block_e8_hierarchy(orc):
    """The E8 hierarchy with two blocks: parents per block (R27, R28)."""
    rng = np.random.default_rng(7)
    X = (rng.standard_normal((3000, 24)) * 0.5).astype(np.float32)
    Q = (X[:25] + 0.05 * rng.standard_normal((25, 24))).astype(np.float32)
    ix = orc.OracleIndex(X, G=2, M=16, W=1.0, seed=3, quantizer=1)
    ix.query(Q, 10, probe=2, T=8, hierarchy=1, min_cand=200)
    base, lvl, ql, code = ix.get("q_base"), ix.get("q_level"), ix.get("q_leaf"), ix.get("q_code")
    uleaf, uoff, perm, pcode = ix.get("uleaf"), ix.get("uoff"), ix.get("perm"), ix.get("code")

    def chain(c, j):
        for _ in range(j):
            c = np.concatenate([orc.e8_parent(c[:8]), orc.e8_parent(c[8:])])
        return c

    seen = set()
    for q in range(len(Q)):
        if base[q] >= 200 or lvl[q] > 32:
            continue
        L = int(lvl[q])
        seen.add(L)
        bks = np.nonzero(uleaf == ql[q])[0]
        node = [u for u in bks if np.array_equal(chain(pcode[perm[uoff[u]]], L), chain(code[q], L))]
        assert node and sum(int(uoff[u + 1] - uoff[u]) for u in node) >= 200
    assert seen
