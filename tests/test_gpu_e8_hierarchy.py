"""GPU parity for the E8 code hierarchy (Eq. 10; reading R27):
per-query level and tau, candidate sets (A0 u node, deduplicated lists)
bit-exact against the oracle; distances within 1e-5, ids equal except ties."""
import numpy as np
import pytest

import synth
from parity_utils import check_topk
from test_gpu_parity import build_pair

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


def gpu_list_candidates(ix, nq):
    off = ix.export("Q_CAND_OFF")
    ids = ix.export("Q_CAND")
    return [ids[off[q]:off[q + 1]] for q in range(nq)]


def run_e8h(ix, ox, X, Q, k, probe, T, tau):
    Qd = torch.from_numpy(Q).cuda()
    ids, d2, nc = ix.query(Qd, k, probe=probe, n_probes=T, hierarchy=1, min_cand=tau, keep_stages=True)
    torch.cuda.synchronize()
    ids, d2, nc = ids.cpu().numpy(), d2.cpu().numpy(), nc.cpu().numpy()
    oi, od, onc = ox.query(Q, k, probe=probe, T=T, hierarchy=1, min_cand=tau)
    assert int(ix.export("Q_TAU")[0]) == ox.tau
    assert np.array_equal(ix.export("Q_BASE"), ox.get("q_base"))
    assert np.array_equal(ix.export("Q_LEVEL"), ox.get("q_level")), "hierarchy level differs"
    gc = gpu_list_candidates(ix, len(Q))
    oc = ox.candidates()
    for q in range(len(Q)):
        assert np.array_equal(gc[q], oc[q]), f"candidate set of query {q} differs"
    assert np.array_equal(nc, onc)
    check_topk(ids, d2, oi, od, X, Q, cands=oc)
    return ox.get("q_level")


@pytest.mark.parametrize("W", [1.0, 2.0, 4.0])
def test_e8_hierarchy(blsh, orc, c1, W):
    X, Q = c1
    ix, ox = build_pair(blsh, orc, X, G=4, M=8, W=W, seed=42, quantizer=1)
    levels = set()
    for probe, T in [(0, 1), (2, 4)]:
        for tau in (0, 400, 2000):
            levels |= set(run_e8h(ix, ox, X, Q, 10, probe, T, tau).tolist())
    assert len(levels) >= 3          # several hierarchy levels exercised


def test_e8_hierarchy_large_k_and_shapes(blsh, orc):
    rng = np.random.default_rng(3)
    X = (rng.standard_normal((4000, 40)) * np.repeat(rng.random((20, 1)) + 0.2, 200, axis=0)).astype(np.float32)
    Q = (X[rng.choice(4000, 60, replace=False)] + 0.05 * rng.standard_normal((60, 40))).astype(np.float32)
    ix, ox = build_pair(blsh, orc, X, G=8, M=8, W=1.5, seed=5, quantizer=1)
    run_e8h(ix, ox, X, Q, 100, 2, 8, 0)
    run_e8h(ix, ox, X, Q, 10, 2, 241, 300)


def test_e8_hierarchy_sharded_global_median(blsh, orc, c1):
    X, Q = c1
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    full = blsh.blsh_build(Xd, n_leaves=4, M=8, W=2.0, seed=42, quantizer=1)
    i1, d1, n1 = full.query(Qd, 10, probe=2, n_probes=4, hierarchy=1)
    shards = [blsh.blsh_build(Xd, n_leaves=4, M=8, W=2.0, seed=42, quantizer=1, rank=r, world=2) for r in range(2)]
    gb = sum(sh.base_counts(Qd, probe=2, n_probes=4) for sh in shards)
    parts, ncs = [], []
    for sh in shards:
        pk, nc = sh.query_packed(Qd, 10, probe=2, n_probes=4, hierarchy=1, global_base=gb)
        parts.append(pk)
        ncs.append(nc)
    mi, md = blsh.blsh_merge_topk(torch.cat(parts).contiguous(), 2, len(Q), 10)
    torch.cuda.synchronize()
    assert torch.equal(mi, i1) and torch.equal(md.view(torch.int32), d1.view(torch.int32))
    assert torch.equal(ncs[0] + ncs[1], n1)


@pytest.mark.parametrize("T", [242, 250, 256])
def test_recursive_e8_probing(blsh, orc, c1, T):
    """after the 240 neighbours, the second ring (R26), probe keys and
    candidate sets bit-exact, with and without the hierarchy."""
    from test_gpu_parity import run_query_pair
    X, Q = c1
    ix, ox = build_pair(blsh, orc, X, G=4, M=8, W=1.0, seed=42, quantizer=1)
    run_query_pair(ix, ox, X, Q, 10, probe=2, T=T)
    run_e8h(ix, ox, X, Q, 10, 2, T, 0)


def test_two_block_e8(blsh, orc):
    """M = 16: two E8 blocks (R28) -- build, lattice probes over 480
    one-block moves, the hierarchy with per-block parents."""
    from test_gpu_parity import compare_build, run_query_pair
    rng = np.random.default_rng(6)
    X = (rng.standard_normal((3000, 24)) * 0.5).astype(np.float32)
    Q = (X[:40] + 0.05 * rng.standard_normal((40, 24))).astype(np.float32)
    ix, ox = build_pair(blsh, orc, X, G=2, M=16, W=1.0, seed=3, quantizer=1)
    compare_build(ix, ox)
    run_query_pair(ix, ox, X, Q, 10, probe=0, T=1)
    run_query_pair(ix, ox, X, Q, 10, probe=2, T=40)
    run_query_pair(ix, ox, X, Q, 100, probe=2, T=256)
    run_e8h(ix, ox, X, Q, 10, 2, 8, 200)
    run_e8h(ix, ox, X, Q, 10, 0, 1, 0)
