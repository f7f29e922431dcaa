"""GPU: queries with NaN / Inf coordinates (reading R30).

A non-finite projection has no probe order (its multiprobe / lattice scores
are NaN), so such a query gets no probes and no candidates: padding rows and
|A(q)| = 0, on both sides.  The other queries of the batch are unaffected.
The point of the test is that the CUDA path never indexes past its selection
(warp_select over an all-NaN pool) and agrees with the oracle on
every finite query, bit for bit on probe keys and candidate sets.
"""
import numpy as np
import pytest

import synth
from parity_utils import check_topk, gpu_candidates

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def blsh():
    if not torch.cuda.is_available():
        pytest.skip("needs CUDA")
    from paper_conf_icde_panm12_b200 import blsh as b
    b.lib()
    return b


def _queries(Q):
    Q = Q.copy()
    Q[3, 0] = np.nan
    Q[7, 5] = np.inf
    Q[11, :] = -np.inf
    Q[20, 17] = np.nan
    return Q, [3, 7, 11, 20]


@pytest.mark.parametrize("quantizer,probe,T,hier", [(0, 1, 16, 0), (0, 1, 240, 0), (0, 1, 8, 1), (0, 0, 1, 1),
                                                     (0, 3, 6, 0), (1, 2, 16, 0), (1, 2, 250, 0), (1, 2, 8, 1)])
def test_nonfinite_queries(blsh, orc, quantizer, probe, T, hier):
    X, Q0 = synth.make_dataset(synth.CONFIGS["c1"])
    Q, bad = _queries(Q0)
    W = 4.0
    ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=4, M=8, W=W, seed=42, quantizer=quantizer,
                         keep_stages=True)
    ox = orc.OracleIndex(X, G=4, M=8, W=W, seed=42, quantizer=quantizer)
    k = 10
    ids, d2, nc = ix.query(torch.from_numpy(Q).cuda(), k, probe=probe, n_probes=T, hierarchy=hier, keep_stages=True)
    torch.cuda.synchronize()
    ids, d2, nc = ids.cpu().numpy(), d2.cpu().numpy(), nc.cpu().numpy()
    oi, od, onc = ox.query(Q, k, probe=probe, T=T, hierarchy=hier)
    assert np.array_equal(ix.export("Q_OOR"), ox.get("q_oor"))
    for q in bad:
        assert ix.export("Q_OOR")[q] & 4, f"query {q}: non-finite flag not set"
        assert nc[q] == 0 and onc[q] == 0
        assert np.all(ids[q] == -1) and np.all(np.isinf(d2[q]))
    assert np.array_equal(ix.export("Q_PVALID"), ox.get("q_pvalid").ravel())
    assert np.array_equal(ix.export("Q_PKEY"), ox.get("q_pkey").ravel())
    if quantizer == 1 and hier:   # E8 code hierarchy: candidates as deduplicated lists (list path)
        off, lst = ix.export("Q_CAND_OFF"), ix.export("Q_CAND")
        gc = [np.sort(lst[off[q]:off[q + 1]]) for q in range(len(Q))]
    else:
        gc = gpu_candidates(ix, T)
    oc = ox.candidates()
    for q in range(len(Q)):
        assert np.array_equal(gc[q], oc[q]), f"candidate set of query {q} differs"
    assert np.array_equal(nc, onc)
    good = np.array([q for q in range(len(Q)) if q not in bad])
    check_topk(ids[good], d2[good], oi[good], od[good], X, Q[good], cands=[oc[q] for q in good])
