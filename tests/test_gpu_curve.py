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
    monkeypatch.setenv("BLSH_SHORTLIST", mode)   # (tc: forced; 100 queries would take the warp list)
    run_query_pair(*c1_pair_w1, X, Q, 10, probe=3, T=6)
    assert c1_pair_w1[0].stats().tiled == {"warp": 0, "simt": 1, "tc": 2}[mode]


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


# P:132's remaining parts: bit-perturbed repeats of the curve search (R31) and the
# shared-MSB climb (R32), bit-exact against the oracle (probe keys, validity, levels,
# candidate sets), distances within 1e-5.

@pytest.mark.parametrize("P,T", [(1, 4), (3, 8), (8, 18), (8, 256), (2, 33)])
@pytest.mark.parametrize("k", [10, 50])
def test_curve_perturbed(c1_pair_w1, c1, P, T, k):
    X, Q = c1
    run_query_pair(*c1_pair_w1, X, Q, k, probe=3, T=T, curve_perturb=P)


@pytest.mark.parametrize("W,msb_min,probe,T", [(1.0, 0, 0, 1), (1.0, 0, 1, 4), (1.0, 112, 3, 3), (1.0, 124, 3, 5)])
def test_msb_climb(blsh, orc, c1, W, msb_min, probe, T):
    X, Q = c1
    ix, ox = build_pair(blsh, orc, X, G=4, M=8, W=W, seed=42)
    run_query_pair(ix, ox, X, Q, 10, probe=probe, T=T, hierarchy=2, msb_min=msb_min)


def test_msb_climb_with_perturbed_curve(c1_pair_w1, c1):
    X, Q = c1
    run_query_pair(*c1_pair_w1, X, Q, 10, probe=3, T=6, hierarchy=2, curve_perturb=2)


def test_msb_climb_low_density_queries(blsh, orc):
    """C3-shaped data with between-cluster queries (P:129 low-density regions): the climb
    triggers for many queries; M = 6 keys (B*M = 96 < 128 bits)."""
    cfg = synth.CONFIGS["c3"]
    from dataclasses import replace
    cfg = replace(cfg, n=20000, nq=300, backend="numpy")
    X, Q = synth.make_dataset(cfg)
    ix, ox = build_pair(blsh, orc, X, G=8, M=6, W=0.6, seed=7)
    _, _, nc = run_query_pair(ix, ox, X, Q, 20, probe=3, T=2, hierarchy=2, curve_perturb=3)
    assert (ix.export("Q_LEVEL") > 0).sum() > 10


def test_perturb_and_climb_rejected(blsh, c1):
    X, Q = c1
    Xd, Qd = torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda()
    ix = blsh.blsh_build(Xd, n_leaves=4, M=8, W=1.0)
    with pytest.raises(blsh.BlshError):
        ix.query(Qd, 10, probe=1, n_probes=4, curve_perturb=1)
    with pytest.raises(blsh.BlshError):
        ix.query(Qd, 10, probe=3, n_probes=4, curve_perturb=9)
    with pytest.raises(blsh.BlshError):
        ix.query(Qd, 10, hierarchy=2, msb_min=129)
    e8 = blsh.blsh_build(Xd, n_leaves=4, quantizer=1)
    with pytest.raises(blsh.BlshError):
        e8.query(Qd, 10, hierarchy=2)
