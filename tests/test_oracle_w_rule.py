"""Oracle pins for the per-leaf width rule (W_rule = 1; "we may choose
different LSH parameters (e.g. bucket size W) that are optimal for each cell";
reading R29: W_g = W sqrt(D_g / D_med), D_g = Delta_A^2 of leaf g)."""
import numpy as np

import synth


def _leaf_D(X, leaf, G):
    D = np.zeros(G)
    for g in range(G):
        m = X[leaf == g].astype(np.float64)
        if len(m):
            mu = m.mean(0)
            D[g] = 2.0 * ((m - mu) ** 2).sum(1).mean()
    return D


def test_w_rule_widths(orc):
    X, _ = synth.make_dataset(synth.CONFIGS["c1"])
    G, W = 8, 3.0
    ix = orc.OracleIndex(X, G=G, M=8, W=W, seed=5, W_rule=1)
    Wl = ix.get("W")
    D = _leaf_D(X, ix.get("leaf"), G)
    med = np.sort(D)[(G - 1) // 2]
    want = W * np.sqrt(D / med)
    assert np.allclose(Wl, want, rtol=1e-6)
    assert np.any(Wl == np.float32(W))                         # the median leaf keeps W exactly
    # the tree does not depend on the widths; (a, b) are the R2 draws with the new widths
    base = orc.OracleIndex(X, G=G, M=8, W=W, seed=5)
    assert np.array_equal(ix.get("theta"), base.get("theta")) and np.array_equal(ix.get("leaf"), base.get("leaf"))
    A, b, _, _ = orc.gen_params(5, G, 8, X.shape[1], Wl)
    assert np.array_equal(ix.get("A"), A) and np.array_equal(ix.get("b"), b)
    assert np.all((b >= 0) & (b < Wl[:, None]))


def test_w_rule_adapts_to_density(orc):
    """Two clusters with spreads 1 : 5 split by the root: the widths follow the spread."""
    rng = np.random.default_rng(3)
    _, _, dirs, _ = orc.gen_params(1, 2, 4, 16, 2.0)
    u = dirs[0].astype(np.float64)                 # the root's RP direction: centres on either side of it
    a = rng.standard_normal((2000, 16)) * 0.2 + 10.0 * u
    b = rng.standard_normal((2000, 16)) * 1.0 - 10.0 * u
    X = np.concatenate([a, b]).astype(np.float32)
    ix = orc.OracleIndex(X, G=2, M=4, W=2.0, seed=1, W_rule=1)
    Wl, leaf = ix.get("W"), ix.get("leaf")
    tight = int(np.bincount(leaf[:2000], minlength=2).argmax())
    assert 4.0 < Wl[1 - tight] / Wl[tight] < 6.0


def test_w_rule_rejects_w_leaf(orc):
    import pytest
    X, _ = synth.make_dataset(synth.CONFIGS["c1"])
    with pytest.raises(orc.OracleError):
        orc.OracleIndex(X, G=4, W=2.0, W_rule=1, W_leaf=np.ones(4, np.float32))
