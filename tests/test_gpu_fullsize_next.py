"""GPU parity at full size for the SURVEY §8(f) rows, in the launch
configuration bench.py times (the whole batch on the GPU, checked on a sample
the oracle answers).

p217 (the paper's evaluation setting: 100k items, 100k queries, L = 10
tables, M = 8, k = 500, standard probing): every table's directory bit for
bit, then the sampled queries' candidate sets (union over the 10 tables),
counts and top-500 lists.

c3 with the E8 index (lattice probing T = 16 + the E8 code hierarchy, P:147,
P:162-173): tau is the batch median, so the oracle answers the sample with the
GPU's tau as an explicit threshold (the median itself is checked against the
oracle's base counts of the whole batch).
"""
from dataclasses import replace

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


def _list_candidates(ix, nq):
    off = ix.export("Q_CAND_OFF")
    ids = ix.export("Q_CAND")
    return [ids[off[q]:off[q + 1]] for q in range(nq)]


def test_p217_full_size(blsh, orc):
    cfg = synth.CONFIGS["p217"]
    Xd, Qd = synth.make_dataset(cfg, backend="torch", device="cuda")
    X, Q = Xd.cpu().numpy(), Qd.cpu().numpy()
    ix = blsh.blsh_build(Xd, n_leaves=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index, n_tables=cfg.L)
    ids, d2, nc = ix.query(Qd, cfg.k, probe=cfg.probe, n_probes=cfg.T)
    torch.cuda.synchronize()
    ids, d2, nc = ids.cpu().numpy(), d2.cpu().numpy(), nc.cpu().numpy()
    ox = orc.OracleIndex(X, G=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index, L=cfg.L)
    for l in range(cfg.L):
        for g, o in [("PERM", "perm"), ("UKEY", "ukey"), ("UOFF", "uoff"), ("LEAF_U", "leaf_u")]:
            assert np.array_equal(ix.export(g, table=l), ox.get(o, l).ravel()), f"table {l}: {g} differs"
    rng = np.random.default_rng(5)
    sample = np.sort(rng.choice(len(Q), 200, replace=False))
    oi, od, onc = ox.query(Q[sample], cfg.k, probe=cfg.probe, T=cfg.T)
    assert np.array_equal(nc[sample], onc), "|A(q)| differs"
    # candidate sets of the sample (same index, same arithmetic: a sub-batch has the same lists)
    ix.query(torch.from_numpy(Q[sample]).cuda(), cfg.k, probe=cfg.probe, n_probes=cfg.T, keep_stages=True)
    gc = _list_candidates(ix, len(sample))
    oc = ox.candidates()
    for i in range(len(sample)):
        assert np.array_equal(gc[i], oc[i]), f"candidate set of query {sample[i]} differs"
    check_topk(ids[sample], d2[sample], oi, od, X, Q[sample], cands=oc)


def test_c3_e8_hierarchy_full_size(blsh, orc):
    cfg = replace(synth.CONFIGS["c3"], quantizer=1, probe=2, T=16, hierarchy=1)
    Xd, Qd = synth.make_dataset(cfg, backend="torch", device="cuda")
    X, Q = Xd.cpu().numpy(), Qd.cpu().numpy()
    ix = blsh.blsh_build(Xd, n_leaves=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index, quantizer=1)
    ids, d2, nc = ix.query(Qd, cfg.k, probe=2, n_probes=cfg.T, hierarchy=1, keep_stages=True)
    torch.cuda.synchronize()
    ids, d2, nc = ids.cpu().numpy(), d2.cpu().numpy(), nc.cpu().numpy()
    tau = int(ix.export("Q_TAU")[0])
    base = ix.export("Q_BASE")
    level = ix.export("Q_LEVEL")
    ox = orc.OracleIndex(X, G=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index, quantizer=1)
    for g, o in [("PERM", "perm"), ("UKEY", "ukey"), ("UOFF", "uoff"), ("LEAF_U", "leaf_u")]:
        assert np.array_equal(ix.export(g), ox.get(o).ravel()), f"{g} differs at full size"
    # the batch median tau from the oracle's base counts of the whole batch
    ox.query(Q, 1, probe=2, T=cfg.T)
    ob = ox.get("q_base")
    assert np.array_equal(base, ob), "|A0(q)| differs"
    assert tau == int(np.sort(ob)[(len(ob) - 1) // 2]), "batch-median tau differs"
    rng = np.random.default_rng(9)
    sample = np.sort(rng.choice(len(Q), 150, replace=False))
    oi, od, onc = ox.query(Q[sample], cfg.k, probe=2, T=cfg.T, hierarchy=1, min_cand=tau)
    assert np.array_equal(level[sample], ox.get("q_level")), "hierarchy levels differ"
    assert np.array_equal(nc[sample], onc), "|A(q)| differs"
    ix.query(torch.from_numpy(Q[sample]).cuda(), cfg.k, probe=2, n_probes=cfg.T, hierarchy=1, min_cand=tau,
             keep_stages=True)
    gc = _list_candidates(ix, len(sample))
    oc = ox.candidates()
    for i in range(len(sample)):
        assert np.array_equal(gc[i], oc[i]), f"candidate set of query {sample[i]} differs"
    check_topk(ids[sample], d2[sample], oi, od, X, Q[sample], cands=oc)
    assert len(set(level[sample].tolist())) >= 2
