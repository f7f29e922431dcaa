"""GPU parity for L > 1 hash tables (reading R24): per-table parameters,
tables and per-query stages bit-exact against the oracle's table-l indexes,
candidate sets (union over tables) bit-exact, distances within 1e-5, ids
equal except ties."""
import numpy as np
import pytest

import synth
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


@pytest.fixture(scope="module")
def c1():
    return synth.make_dataset(synth.CONFIGS["c1"])


def build_pair(blsh, orc, X, L, G=4, M=8, W=4.0, seed=42, quantizer=0):
    ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=G, M=M, W=W, seed=seed, quantizer=quantizer,
                         keep_stages=True, n_tables=L)
    ox = orc.OracleIndex(X, G=G, M=M, W=W, seed=seed, quantizer=quantizer, L=L)
    assert ix.info().n_tables == L
    for l in range(L):
        for a, b in [("A", "A"), ("B", "b"), ("PERM", "perm"), ("UKEY", "ukey"), ("ULEAF", "uleaf"),
                     ("UOFF", "uoff"), ("LEAF_U", "leaf_u")]:
            g = ix.export(a, table=l)
            o = ox.get(b, l).ravel()
            assert g.shape == o.shape and np.array_equal(g.view(np.uint8), o.view(np.uint8)), f"table {l}: {a}"
    return ix, ox


def gpu_union_candidates(ix, L, T, nq):
    per = []
    for l in range(L):
        iv = ix.export("Q_INTERVALS", table=l).reshape(nq, T + 1, 2)
        perm = ix.export("PERM", table=l)
        per.append([np.concatenate([perm[s:e] for s, e in iv[q] if e > s] or [np.zeros(0, np.int64)])
                    for q in range(nq)])
    return [np.unique(np.concatenate([p[q] for p in per])) for q in range(nq)]


def run_pair(ix, ox, X, Q, k, L, probe=0, T=1):
    Qd = torch.from_numpy(Q).cuda()
    ids, d2, nc = ix.query(Qd, k, probe=probe, n_probes=T, keep_stages=True)
    torch.cuda.synchronize()
    ids, d2, nc = ids.cpu().numpy(), d2.cpu().numpy(), nc.cpu().numpy()
    oi, od, onc = ox.query(Q, k, probe=probe, T=T)
    assert np.array_equal(ix.export("Q_LEAF"), ox.get("q_leaf")), "query leaf differs"
    for l in range(L):
        for a, b in [("Q_T", "q_t"), ("Q_CODE", "q_code"), ("Q_OOR", "q_oor"), ("Q_KEY", "q_key"),
                     ("Q_PKEY", "q_pkey"), ("Q_PVALID", "q_pvalid"), ("Q_BASE", "q_base")]:
            g = ix.export(a, table=l)
            o = ox.get(b, l).ravel()
            assert np.array_equal(g.view(np.uint8), o.view(np.uint8)), f"table {l}: {a} differs"
    gc = gpu_union_candidates(ix, L, T, len(Q))
    oc = ox.candidates()
    for q in range(len(Q)):
        assert np.array_equal(gc[q], oc[q]), f"candidate set of query {q} differs"
    assert np.array_equal(nc, onc)
    check_topk(ids, d2, oi, od, X, Q, cands=oc)
    return ids, d2, nc


@pytest.mark.parametrize("L,probe,T,k", [(2, 0, 1, 10), (3, 0, 1, 64), (4, 1, 8, 10), (3, 1, 16, 100)])
def test_tables_zm(blsh, orc, c1, L, probe, T, k):
    X, Q = c1
    ix, ox = build_pair(blsh, orc, X, L)
    run_pair(ix, ox, X, Q, k, L, probe=probe, T=T)


def test_tables_e8_lattice(blsh, orc, c1):
    X, Q = c1
    ix, ox = build_pair(blsh, orc, X, 2, quantizer=1)
    run_pair(ix, ox, X, Q, 10, 2, probe=2, T=16)


@pytest.mark.parametrize("G,M,W,d", [(1, 8, 2.0, 64), (8, 4, 1.5, 61), (2, 6, 0.8, 17)])
def test_tables_shapes(blsh, orc, G, M, W, d):
    rng = np.random.default_rng(G * 100 + d)
    X = rng.standard_normal((3000, d)).astype(np.float32)
    Q = (X[rng.choice(3000, 50, replace=False)] + 0.05 * rng.standard_normal((50, d))).astype(np.float32)
    ix, ox = build_pair(blsh, orc, X, 3, G=G, M=M, W=W, seed=9)
    run_pair(ix, ox, X, Q, 10, 3, probe=1, T=6)


def test_tables_recall_not_below_single(blsh, c1):
    """Union semantics: more tables -> a superset of candidates."""
    X, Q = c1
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    n_prev = None
    for L in (1, 2, 4):
        ix = blsh.blsh_build(Xd, n_leaves=4, M=8, W=2.0, seed=42, n_tables=L)
        _, _, nc = ix.query(Qd, 10)
        nc = nc.cpu().numpy()
        if n_prev is not None:
            assert np.all(nc >= n_prev)
        n_prev = nc


def test_tables_sharded_merge_matches_single(blsh, c1):
    X, Q = c1
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    full = blsh.blsh_build(Xd, n_leaves=4, M=8, W=4.0, seed=42, n_tables=3)
    i1, d1, n1 = full.query(Qd, 10, probe=1, n_probes=4)
    parts, ncs = [], []
    for r in range(2):
        sh = blsh.blsh_build(Xd, n_leaves=4, M=8, W=4.0, seed=42, rank=r, world=2, n_tables=3)
        pk, nc = sh.query_packed(Qd, 10, probe=1, n_probes=4)
        parts.append(pk)
        ncs.append(nc)
    mi, md = blsh.blsh_merge_topk(torch.cat(parts).contiguous(), 2, len(Q), 10)
    torch.cuda.synchronize()
    assert torch.equal(mi, i1) and torch.equal(md.view(torch.int32), d1.view(torch.int32))
    assert torch.equal(ncs[0] + ncs[1], n1)


def test_tables_rejects_hierarchy(blsh, c1):
    X, Q = c1
    ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=4, n_tables=2)
    with pytest.raises(Exception):
        ix.query(torch.from_numpy(Q).cuda(), 10, hierarchy=1)
    with pytest.raises(Exception):
        blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=4, n_tables=65)
