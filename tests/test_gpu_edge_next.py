"""Edge cases of the next-row paths (L > 1, E8 hierarchy, large k, curve probing,
W_rule, leaf_split): empty batches, tiny and degenerate indexes, against the oracle."""
import numpy as np
import pytest

from parity_utils import check_topk

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def blsh():
    if not torch.cuda.is_available():
        pytest.skip("needs CUDA")
    from paper_conf_icde_panm12_b200 import blsh as b
    b.lib()
    return b


@pytest.mark.parametrize("kw,qkw", [
    (dict(n_tables=3), dict(k=10)),
    (dict(quantizer=1), dict(k=10, probe=2, n_probes=8, hierarchy=1)),
    (dict(), dict(k=300)),
    (dict(), dict(k=10, probe=3, n_probes=5)),
    (dict(W_rule=1, n_tables=2), dict(k=70, probe=1, n_probes=4)),
])
def test_next_paths_edge_cases(blsh, orc, kw, qkw):
    rng = np.random.default_rng(0)
    d = 24
    X = rng.standard_normal((700, d)).astype(np.float32)
    X[100:200] = X[0]                                   # a block of duplicates (ties by id)
    Q = np.concatenate([X[:5], rng.standard_normal((20, d)).astype(np.float32) * 3]).astype(np.float32)
    G = 4
    ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=G, M=8, W=2.0, seed=3, **kw)
    okw = {"L": kw.get("n_tables", 1), "quantizer": kw.get("quantizer", 0), "W_rule": kw.get("W_rule", 0)}
    ox = orc.OracleIndex(X, G=G, M=8, W=2.0, seed=3, **okw)
    k = qkw.pop("k")
    # empty batch
    e = ix.query(torch.zeros((0, d), device="cuda"), k, **qkw)
    assert e[0].shape == (0, k)
    ids, d2, nc = ix.query(torch.from_numpy(Q).cuda(), k, **qkw)
    torch.cuda.synchronize()
    oq = dict(probe=qkw.get("probe", 0), T=qkw.get("n_probes", 1), hierarchy=qkw.get("hierarchy", 0))
    oi, od, onc = ox.query(Q, k, **oq)
    assert np.array_equal(nc.cpu().numpy(), onc)
    check_topk(ids.cpu().numpy(), d2.cpu().numpy(), oi, od, X, Q, cands=ox.candidates())


def test_tables_single_point_leaves(blsh, orc):
    """G = 8 leaves over 9 points: near-empty leaves, L = 2, k larger than any bucket."""
    rng = np.random.default_rng(1)
    X = rng.standard_normal((9, 8)).astype(np.float32)
    Q = rng.standard_normal((6, 8)).astype(np.float32)
    ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=8, M=4, W=1.0, seed=2, n_tables=2)
    ox = orc.OracleIndex(X, G=8, M=4, W=1.0, seed=2, L=2)
    ids, d2, nc = ix.query(torch.from_numpy(Q).cuda(), 100, probe=1, n_probes=9)
    torch.cuda.synchronize()
    oi, od, onc = ox.query(Q, 100, probe=1, T=9)
    assert np.array_equal(nc.cpu().numpy(), onc)
    check_topk(ids.cpu().numpy(), d2.cpu().numpy(), oi, od, X, Q, cands=ox.candidates())
