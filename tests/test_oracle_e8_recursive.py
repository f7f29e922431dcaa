"""Oracle pins for candidate-count-triggered recursive E8 probing ("If the number
of candidates computed is not enough, we recursively probe the adjacent buckets of the
240 probed buckets"; reading R33 in DESIGN.md): with min_cand = tau > 0 and no hierarchy,
the home bucket and the 240 roots are always probed (as with T <= 241), and the second
ring's probes (R26 order) are added one at a time only while the candidates gathered
number fewer than tau.

The pins come from outside the oracle's probe loop: the unconditional runs with T = 241
and T = 256 (two other calls), and every probe bucket's size looked up in numpy from the
exported table (sorted bucket keys and offsets):
  * prefix: the taken probes are the first ones of the T = 256 sequence (same keys);
  * A(T = 241) <= A(tau) <= A(T = 256);
  * sufficiency: |A(tau)| >= min(tau, |A(T = 256)|);
  * minimality: without its last second-ring bucket, A(tau) has fewer than tau points;
  * tau above every count gives T = 256; tau = 1 gives T = 241 wherever A(T=241) is non-empty.
"""
import numpy as np
import pytest

import synth

T_FULL = 256


@pytest.fixture(scope="module")
def e8case(orc):
    cfg = synth.CONFIGS["c1"]
    X, Q = synth.make_dataset(cfg, n=6000, nq=80)
    # narrow cells: few points per bucket, so the 241 first probes often hold few candidates
    ox = orc.OracleIndex(X, G=2, M=8, W=1.2, seed=3, quantizer=1)
    return ox, X, Q


def _run(ox, Q, T, tau):
    ox.query(Q, 10, probe=2, T=T, min_cand=tau)
    return ox.candidates(), ox.get("q_pkey").reshape(len(Q), T, 2), ox.get("q_pvalid").reshape(len(Q), T)


def _bucket_sizes(ox, pkey, pvalid, qleaf):
    """|bucket| of every probe key, by binary search in the exported sorted table."""
    ukey = ox.get("ukey").reshape(-1, 2)
    uleaf = ox.get("uleaf")
    uoff = ox.get("uoff")
    keys = [(int(h) << 64) | int(l) for h, l in ukey]
    out = np.zeros(pvalid.shape, np.int64)
    for q in range(pvalid.shape[0]):
        g = qleaf[q]
        lo, hi = np.searchsorted(uleaf, g, "left"), np.searchsorted(uleaf, g, "right")
        for p in range(pvalid.shape[1]):
            if not pvalid[q, p]:
                continue
            kq = (int(pkey[q, p, 0]) << 64) | int(pkey[q, p, 1])
            a, b = lo, hi
            while a < b:
                m = (a + b) // 2
                if keys[m] < kq:
                    a = m + 1
                else:
                    b = m
            if a < hi and keys[a] == kq:
                out[q, p] = int(uoff[a + 1]) - int(uoff[a])
    return out


def test_recursive_probing_pins(e8case):
    ox, X, Q = e8case
    a241, _, _ = _run(ox, Q, 241, 0)
    afull, kfull, vfull = _run(ox, Q, T_FULL, 0)
    qleaf = ox.get("q_leaf")
    sizes = _bucket_sizes(ox, kfull, vfull, qleaf)
    n241 = np.array([len(a) for a in a241])
    nfull = np.array([len(a) for a in afull])
    # sanity of the independent bucket sizes: they add up to the unconditional counts
    assert np.array_equal(sizes.sum(1), nfull)
    assert np.array_equal(sizes[:, :241].sum(1), n241)
    taus = sorted({1, int(np.median(n241)) + 1, int(np.percentile(nfull, 75)) + 1, int(nfull.max()) + 1})
    triggered = 0
    for tau in taus:
        arec, krec, vrec = _run(ox, Q, T_FULL, tau)
        for q in range(len(Q)):
            A = arec[q]
            # prefix of the T = 256 sequence: same keys where taken, taken -> valid in the full run
            taken = vrec[q] != 0
            assert np.array_equal(taken[:241], vfull[q, :241] != 0)
            assert np.all(~taken | (vfull[q] != 0))
            assert np.array_equal(krec[q][taken], kfull[q][taken])
            ring = np.nonzero(taken[241:])[0] + 241
            if len(ring):
                last = ring[-1]
                # every valid ring probe before the last taken one is taken
                assert np.all(taken[241:last + 1] | (vfull[q, 241:last + 1] == 0))
            assert set(a241[q]).issubset(A) and set(A).issubset(afull[q])
            assert len(A) >= min(tau, len(afull[q]))
            if len(ring):
                triggered += 1
                assert len(A) - sizes[q, ring[-1]] < tau, "a ring probe was taken although tau was reached"
            if tau == 1 and n241[q] > 0:
                assert len(ring) == 0 and np.array_equal(A, a241[q])
            if tau > nfull.max():
                assert np.array_equal(A, afull[q])
    assert triggered > 0, "no query reached the second ring: the pins would not exercise R33"


def test_recursive_probing_needs_tau_and_no_hierarchy(e8case):
    ox, X, Q = e8case
    a0, _, _ = _run(ox, Q, T_FULL, 0)                 # tau = 0: every probe (R26 as before)
    ox.query(Q, 10, probe=2, T=T_FULL, hierarchy=1, min_cand=10 ** 9)   # tau serves the hierarchy instead
    assert all(set(a).issubset(b) for a, b in zip(a0, ox.candidates()))
    a_small, _, _ = _run(ox, Q, 200, 10 ** 9)          # T <= 241: nothing to recurse into
    b_small, _, _ = _run(ox, Q, 200, 0)
    assert all(np.array_equal(a, b) for a, b in zip(a_small, b_small))
