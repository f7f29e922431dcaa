"""Oracle pins: generator (R2), parameters, canonical arithmetic
(R1) and the E2LSH hash (Eq. 2, P:241 collision probability)."""
from fractions import Fraction
import math

import numpy as np
import pytest
from scipy import stats


def test_splitmix64_known_answers(orc):
    # Published SplitMix64 outputs for a generator seeded with 0 (Steele,
    # Lea & Flood, OOPSLA 2014 / Vigna's reference C): R(0, 0, i) is the
    # (i+1)-th output of that generator under reading R2.
    expect = [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F, 0xF88BB8A8724C81EC]
    assert [orc.rng_u64(0, 0, i) for i in range(4)] == expect


def test_uniform_and_gauss_moments(orc):
    u = np.array([orc.rng_uniform(7, 3, i) for i in range(20000)])
    assert u.min() >= 0.0 and u.max() < 1.0
    assert stats.kstest(u, "uniform").pvalue > 1e-3
    g = np.array([orc.rng_gauss(7, 5, i) for i in range(20000)])
    assert abs(g.mean()) < 0.03 and abs(g.var() - 1.0) < 0.04
    assert stats.kstest(g, "norm").pvalue > 1e-3


def test_params_distribution_and_ranges(orc):
    G, M, d, W = 4, 8, 64, 3.5
    A, b, dirs, jit = orc.gen_params(42, G, M, d, W)
    assert A.shape == (G, M, d) and b.shape == (G, M) and dirs.shape == (G - 1, d)
    assert stats.kstest(A.ravel().astype(np.float64), "norm").pvalue > 1e-3   # a ~ N(0,1)
    assert np.all(b >= 0) and np.all(b < W)                                  # b ~ U[0,W)
    nrm = np.linalg.norm(dirs.astype(np.float64), axis=1)
    assert np.allclose(nrm, 1.0, atol=1e-6)                                  # unit direction
    assert np.all((jit >= 0) & (jit < 1))
    # leaves / nodes draw independent parameters (R3)
    assert not np.array_equal(A[0], A[1]) and not np.array_equal(dirs[0], dirs[1])
    # different seed -> different parameters; same seed -> identical bits
    A2, *_ = orc.gen_params(43, G, M, d, W)
    A3, *_ = orc.gen_params(42, G, M, d, W)
    assert not np.array_equal(A, A2) and np.array_equal(A, A3)


def test_canonical_dot_exact_on_integers(orc):
    rng = np.random.default_rng(0)
    for _ in range(50):
        d = int(rng.integers(1, 300))
        a = rng.integers(-50, 50, d).astype(np.float32)
        x = rng.integers(-50, 50, d).astype(np.float32)
        exact = int(np.dot(a.astype(np.int64), x.astype(np.int64)))
        assert float(orc.dot_canonical(a, x)) == exact          # |sum| < 2^24: exact in fp32
        e = (a - x).astype(np.int64)
        assert float(orc.dist2_canonical(a, x)) == int(np.dot(e, e))


def test_canonical_dist_within_fp32_bound(orc):
    rng = np.random.default_rng(1)
    for _ in range(100):
        d = int(rng.integers(1, 600))
        x = rng.standard_normal(d).astype(np.float32)
        y = rng.standard_normal(d).astype(np.float32)
        ref = float(np.sum((x.astype(np.float64) - y.astype(np.float64)) ** 2))
        got = float(orc.dist2_canonical(x, y))
        assert abs(got - ref) <= (d + 2) * 2.0 ** -23 * ref + 1e-30


def _exact_t(a, b, W, x):
    s = sum(Fraction(float(ai)) * Fraction(float(xi)) for ai, xi in zip(a, x))
    return (s + Fraction(float(b))) / Fraction(float(W))


def test_hash_matches_exact_floor(orc):
    """Eq. 2: h_i = floor((a_i . v + b_i) / W), against exact rationals."""
    rng = np.random.default_rng(2)
    M, d, W = 8, 48, 2.75
    A = rng.standard_normal((M, d)).astype(np.float32)
    b = (rng.random(M) * W).astype(np.float32)
    n_checked = 0
    for _ in range(200):
        x = (3 * rng.standard_normal(d)).astype(np.float32)
        t, h = orc.hash_point(A, b, W, x)
        for i in range(M):
            te = _exact_t(A[i], b[i], W, x)
            fl = math.floor(te)
            # fp32 chain error bound on the projection (d+2 roundings of magnitude <= sum|a||x|)
            bound = Fraction((d + 4) * 2.0 ** -23) * (sum(abs(Fraction(float(v))) for v in A[i] * x) + abs(Fraction(float(b[i])))) / Fraction(W)
            assert abs(Fraction(float(t[i])) - te) <= bound
            if te - fl > bound and fl + 1 - te > bound:
                assert h[i] == fl
                n_checked += 1
            else:
                assert h[i] in (fl - 1, fl, fl + 1)
    assert n_checked > 1500


def test_hash_integer_exact_case(orc):
    """Integer a, x, b and power-of-two W: every step is exact, h = floor exactly."""
    rng = np.random.default_rng(3)
    M, d, W = 4, 16, 8.0
    A = rng.integers(-5, 6, (M, d)).astype(np.float32)
    b = rng.integers(0, 8, M).astype(np.float32)
    for _ in range(200):
        x = rng.integers(-20, 21, d).astype(np.float32)
        _, h = orc.hash_point(A, b, W, x)
        exact = np.floor_divide(A.astype(np.int64) @ x.astype(np.int64) + b.astype(np.int64), 8)
        assert np.array_equal(h, exact)


def test_collision_probability_closed_form(orc):
    """with b ~ U[0,W), P[h(u) = h(v)] = 1 - min(|a.u - a.v|, W) / W."""
    rng = np.random.default_rng(4)
    d, W = 32, 1.0
    a = rng.standard_normal((1, d)).astype(np.float32)
    u = rng.standard_normal(d).astype(np.float32)
    for scale in (0.0, 0.1, 0.4, 0.8, 1.5):
        v = (u + scale * a[0] / np.linalg.norm(a[0])).astype(np.float32)
        sep = abs(float(np.dot(a[0].astype(np.float64), u - v)))
        p = 1.0 - min(sep, W) / W
        trials = 4000
        hits = 0
        for _ in range(trials):
            b = np.array([rng.random() * W], np.float32)
            hits += int(orc.hash_point(a, b, W, u)[1][0] == orc.hash_point(a, b, W, v)[1][0])
        se = math.sqrt(max(p * (1 - p), 1e-4) / trials)
        assert abs(hits / trials - p) < 5 * se + 2e-3
