"""GPU parity for Morton-curve neighbour probing (probe = 3, R25):
probe keys / validity / candidate sets bit-exact against the oracle,
distances within 1e-5, ids equal except ties; with the hierarchy, the
query-tiled short-lists, L > 1 tables and a sharded index."""
import numpy as np
import pytest

import synth
from test_gpu_parity import build_pair, run_query_pair
from test_gpu_tables import build_pair as build_pair_tables, run_pair as run_pair_tables

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


@pytest.fixture(scope="module")
def c1_pair_w1(blsh, orc, c1):
    X, _ = c1
    return build_pair(blsh, orc, X, G=4, M=8, W=1.0, seed=42)


@pytest.mark.parametrize("T", [1, 2, 7, 33, 256])
@pytest.mark.parametrize("k", [10, 50, 100])
def test_curve_probes(c1_pair_w1, c1, T, k):
    X, Q = c1
    run_query_pair(*c1_pair_w1, X, Q, k, probe=3, T=T)


@pytest.mark.parametrize("mode", ["warp", "simt", "tc"])
def test_curve_shortlist_variants(c1_pair_w1, c1, monkeypatch, mode):
    X, Q = c1
    if mode != "tc":
        monkeypatch.setenv("BLSH_SHORTLIST", mode)
    run_query_pair(*c1_pair_w1, X, Q, 10, probe=3, T=6)


def test_curve_with_hierarchy(c1_pair_w1, c1):
    X, Q = c1
    run_query_pair(*c1_pair_w1, X, Q, 10, probe=3, T=4, hierarchy=1)
    run_query_pair(*c1_pair_w1, X, Q, 10, probe=3, T=2, hierarchy=1, hier_step_bits=1, min_cand=800)


def test_curve_with_tables(blsh, orc, c1):
    X, Q = c1
    ix, ox = build_pair_tables(blsh, orc, X, 3, W=1.5)
    run_pair_tables(ix, ox, X, Q, 10, 3, probe=3, T=5)


def test_curve_sharded(blsh, c1):
    X, Q = c1
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    full = blsh.blsh_build(Xd, n_leaves=4, M=8, W=1.0, seed=42)
    i1, d1, _ = full.query(Qd, 10, probe=3, n_probes=9)
    parts = []
    for r in range(4):
        sh = blsh.blsh_build(Xd, n_leaves=4, M=8, W=1.0, seed=42, rank=r, world=4)
        parts.append(sh.query_packed(Qd, 10, probe=3, n_probes=9)[0])
    mi, md = blsh.blsh_merge_topk(torch.cat(parts).contiguous(), 4, len(Q), 10)
    torch.cuda.synchronize()
    assert torch.equal(mi, i1) and torch.equal(md.view(torch.int32), d1.view(torch.int32))


def test_curve_rejected_on_e8(blsh, c1):
    X, Q = c1
    ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=4, quantizer=1)
    with pytest.raises(blsh.BlshError):
        ix.query(torch.from_numpy(Q).cuda(), 10, probe=3, n_probes=4)
