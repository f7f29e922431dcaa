"""Small batches replayed as CUDA graphs (api.cu query_graph): the first call of a shape runs
normally and is captured, later calls of that shape replay the graph on new inputs.  Every
call must answer like the oracle (counts bit-exact, top-k by check_topk), including a batch
statistic computed inside the graph (the hierarchy's median tau, R18) and the statistics
read back per call."""
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


@pytest.mark.parametrize("kw", [dict(probe=1, T=16), dict(probe=1, T=8, hierarchy=1), dict(probe=0, T=1)])
def test_graph_replays_match_oracle(blsh, orc, kw):
    X, Q = synth.make_dataset(synth.CONFIGS["c1"], n=10000, nq=200)
    ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=4, M=8, W=4.0, seed=21)
    ox = orc.OracleIndex(X, G=4, M=8, W=4.0, seed=21)
    T = kw["T"]
    hk = dict(hierarchy=kw.get("hierarchy", 0))
    for rep in range(2):
        for b in range(3):            # same shape (50 queries), different inputs: capture, then replays
            Qb = Q[50 * b:50 * (b + 1)]
            ids, d2, nc = ix.query(torch.from_numpy(Qb).cuda(), 10, probe=kw["probe"], n_probes=T, **hk)
            torch.cuda.synchronize()
            st = ix.stats()
            ids, d2, nc = ids.cpu().numpy(), d2.cpu().numpy(), nc.cpu().numpy()
            oi, od, onc = ox.query(Qb, 10, probe=kw["probe"], T=T, **hk)
            assert np.array_equal(nc, onc), f"counts differ (rep {rep}, batch {b})"
            check_topk(ids, d2, oi, od, X, Qb, cands=ox.candidates())
            assert st.total_cand == int(onc.sum())
            if hk["hierarchy"]:
                assert st.tau == ox.tau
    ix.close()
