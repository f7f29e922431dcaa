"""Oracle pins: Morton keys (Eq. 7-9), E8 decoding and roots,
multiprobe order (Lv et al. [8] heap method)."""
import heapq
import itertools
import os
from fractions import Fraction

import numpy as np
import pytest

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _rows(name):
    out = []
    for line in open(os.path.join(GOLD, name)):
        line = line.strip()
        if line and not line.startswith("#"):
            out.append(line.split())
    return out


# --- Morton -------------------------------------------------------------------

@pytest.mark.parametrize("M", [1, 2, 3, 5, 8, 16])
def test_morton_roundtrip(orc, M):
    """the Morton code is one-to-one with the LSH code."""
    B = orc.bits_per_coord(M)
    rng = np.random.default_rng(M)
    seen = set()
    for _ in range(300):
        c = rng.integers(-(2 ** (B - 1)), 2 ** (B - 1), M).astype(np.int32)
        k = orc.morton_encode(c)
        assert 0 <= k < 2 ** (B * M)
        assert np.array_equal(orc.morton_decode(k, M), c)
        seen.add((tuple(c), k))
    assert len({k for _, k in seen}) == len(seen)


def test_morton_z_order_golden(orc):
    """Sorting Morton codes visits the 4x4 grid in Z-order."""
    rows = _rows("morton_z2_grid.txt")
    codes = [(int(r[1]), int(r[2])) for r in rows]
    keys = [orc.morton_encode(np.array(c, np.int32)) for c in codes]
    assert keys == sorted(keys) and len(set(keys)) == 16


def test_eq9_golden(orc):
    for x, m, n, want in (map(int, r) for r in _rows("eq9_floor_identity.txt")):
        assert (x // m) // n == x // (m * n) == want


def _ancestor_eq7(c, k):
    """Eq. 7: k-fold floor-halving of every coordinate (PAPER.md 151)."""
    c = list(int(v) for v in c)
    for _ in range(k):
        c = [v // 2 for v in c]
    return tuple(c)


@pytest.mark.parametrize("M", [2, 3, 8])
def test_morton_prefix_is_eq8_ancestor(orc, M):
    """Keys share their top (B-l)*M bits  <=>  same level-l ancestor (Eq. 7-8), l < B."""
    B = orc.bits_per_coord(M)
    rng = np.random.default_rng(10 + M)
    for _ in range(400):
        c1 = rng.integers(-40, 40, M)
        c2 = c1 + rng.integers(-6, 7, M)
        k1 = orc.morton_encode(c1.astype(np.int32))
        k2 = orc.morton_encode(c2.astype(np.int32))
        for lvl in range(0, min(B, 9)):
            same_prefix = (k1 >> (lvl * M)) == (k2 >> (lvl * M))
            assert same_prefix == (_ancestor_eq7(c1, lvl) == _ancestor_eq7(c2, lvl))


# --- E8 -------------------------------------------------------------------------

def _in_e8(p):
    """E8 membership straight from P:138: all integer or all half-integer, even sum."""
    p = [Fraction(float(v)).limit_denominator(4) for v in p]
    ints = all(v.denominator == 1 for v in p)
    halves = all(v.denominator == 2 for v in p)
    return (ints or halves) and sum(p).denominator == 1 and sum(p).numerator % 2 == 0


def test_e8_membership_golden(orc):
    for r in _rows("e8_membership.txt"):
        member = r[0] == "1"
        p = np.array([float(v) for v in r[1:]], np.float32)
        assert _in_e8(p) == member
        c2 = orc.e8_decode(p)
        assert np.array_equal(c2, (2 * p).astype(np.int32)) == member


def test_e8_roots(orc):
    roots = orc.e8_roots()
    assert roots.shape == (240, 8)
    assert len({tuple(r) for r in roots}) == 240
    assert np.all((roots.astype(np.int64) ** 2).sum(1) == 8)           # norm^2 = 2 (doubled: 8)
    assert all(_in_e8(r / 2.0) for r in roots)
    # independent enumeration of all E8 vectors of norm^2 2
    cand = set()
    for vals in itertools.product((-2, -1, 0, 1, 2), repeat=8):
        if sum(v * v for v in vals) == 8 and _in_e8([v / 2.0 for v in vals]):
            cand.add(vals)
    assert cand == {tuple(r) for r in roots}


def test_e8_decode_is_nearest(orc):
    rng = np.random.default_rng(5)
    roots = orc.e8_roots().astype(np.float64) / 2
    for _ in range(400):
        y = (rng.standard_normal(8) * rng.choice([0.3, 1.0, 4.0])).astype(np.float32)
        c2 = orc.e8_decode(y)
        c = c2 / 2.0
        assert _in_e8(c)
        dy = np.sum((y.astype(np.float64) - c) ** 2)
        dn = np.sum((y.astype(np.float64)[None, :] - (c[None, :] + roots)) ** 2, axis=1)
        assert np.all(dy <= dn + 1e-12)          # 240 roots are E8's Voronoi-relevant vectors
    for lp in roots[:20]:
        assert np.array_equal(orc.e8_decode(lp.astype(np.float32)), (2 * lp).astype(np.int32))


def test_e8_decode_brute_force_small(orc):
    rng = np.random.default_rng(6)
    pts = []
    for vals in itertools.product((-2, -1, 0, 1, 2), repeat=8):
        if sum(vals) % 2 == 0:
            pts.append(vals)
    for vals in itertools.product((-1.5, -0.5, 0.5, 1.5), repeat=8):
        if (sum(vals) % 2) == 0:
            pts.append(vals)
    pts = np.array(pts, np.float64)
    for _ in range(100):
        y = rng.uniform(-1, 1, 8).astype(np.float32)
        c = orc.e8_decode(y) / 2.0
        d = np.sum((pts - y.astype(np.float64)) ** 2, axis=1)
        assert np.isclose(np.sum((c - y) ** 2), d.min(), rtol=0, atol=1e-12)


def test_lattice_order_sorted(orc):
    rng = np.random.default_rng(7)
    roots = orc.e8_roots()
    for _ in range(30):
        y = rng.standard_normal(8).astype(np.float32) * 2
        c2 = orc.e8_decode(y)
        idx = orc.lattice_order(y, c2, 241)
        assert sorted(idx.tolist()) == list(range(240))
        sc = [np.sum((y.astype(np.float64) - (c2 + roots[i]) / 2.0) ** 2) for i in idx]
        assert all(sc[i] <= sc[i + 1] for i in range(239))
        assert all(idx[i] < idx[i + 1] for i in range(239) if sc[i] == sc[i + 1])


# --- multiprobe -----------------------------------------------------------------

def _lv_heap(t, T):
    """Lv et al. [8] query-directed probing, heap method (shift / expand), in
    exact rational arithmetic.  Independent of the oracle's enumeration."""
    M = len(t)
    f = [np.floor(np.float32(v)) for v in t]
    xm = [np.float32(np.float32(v) - np.float32(fl)) for v, fl in zip(t, f)]
    xp = [np.float32(np.float32(1.0) - v) for v in xm]
    # 2M (value, coord, sign) sorted by value
    z = sorted([(Fraction(float(xm[i])) ** 2, i, -1) for i in range(M)] +
               [(Fraction(float(xp[i])) ** 2, i, +1) for i in range(M)],
               key=lambda e: (e[0], e[1], e[2]))

    def score(s):
        return sum(z[j][0] for j in s)

    def valid(s):
        coords = [z[j][1] for j in s]
        return len(coords) == len(set(coords))

    out = []
    heap = [(score((0,)), (0,))]
    while heap and len(out) < T - 1:
        sc, s = heapq.heappop(heap)
        if valid(s):
            delta = [0] * M
            for j in s:
                delta[z[j][1]] = z[j][2]
            out.append((sc, tuple(delta)))
        last = s[-1]
        if last + 1 < 2 * M:
            sh = s[:-1] + (last + 1,)
            ex = s + (last + 1,)
            heapq.heappush(heap, (score(sh), sh))
            heapq.heappush(heap, (score(ex), ex))
    return out


@pytest.mark.parametrize("M", [2, 3, 4, 6, 8])
def test_multiprobe_matches_lv_heap(orc, M):
    rng = np.random.default_rng(20 + M)
    for _ in range(25):
        t = (rng.standard_normal(M) * 5).astype(np.float32)
        T = int(min(3 ** M, rng.integers(2, 65)))
        deltas, scores = orc.multiprobe_deltas(t, T)
        ref = _lv_heap(t, T)
        assert len(ref) == T - 1
        ref_scores = [float(s) for s, _ in ref]
        assert np.allclose(scores, ref_scores, rtol=1e-12, atol=0)
        # exact ties are measure-zero here; the sequences must agree
        assert [tuple(d) for d in deltas] == [d for _, d in ref]


def test_multiprobe_properties(orc):
    rng = np.random.default_rng(30)
    M = 8
    for _ in range(20):
        t = (rng.standard_normal(M) * 3).astype(np.float32)
        deltas, scores = orc.multiprobe_deltas(t, 3 ** M)
        assert len({tuple(d) for d in deltas}) == 3 ** M - 1
        assert not any(np.all(d == 0) for d in deltas)
        assert np.all(np.diff(scores) >= 0)
        # first probe: the single coordinate closest to a cell boundary
        f = np.floor(t)
        xm = t - f
        xp = 1 - xm
        best = np.minimum(xm, xp)
        i = int(np.argmin(best))
        assert np.count_nonzero(deltas[0]) == 1 and deltas[0][i] == (-1 if xm[i] <= xp[i] else 1)
    d1, _ = orc.multiprobe_deltas(np.zeros(4, np.float32) + 0.3, 1)
    assert d1.shape[0] == 0
