"""GPU parity for candidate-count-triggered recursive E8 probing (reading R33):
probe keys, validity (probes not taken are invalid), |A0|, candidate sets bit-exact and
top-k against the oracle, for thresholds that stop the recursion at every depth."""
import numpy as np
import pytest

import synth
from test_gpu_parity import build_pair, run_query_pair

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
def e8pair(blsh, orc):
    cfg = synth.CONFIGS["c1"]
    X, Q = synth.make_dataset(cfg, n=6000, nq=80)
    ix, ox = build_pair(blsh, orc, X, G=2, M=8, W=1.2, seed=3, quantizer=1)
    return ix, ox, X, Q


@pytest.mark.parametrize("tau", [1, 30, 120, 400, 10 ** 9])
@pytest.mark.parametrize("T", [250, 256])
def test_recursive_lattice_probing(e8pair, tau, T):
    ix, ox, X, Q = e8pair
    run_query_pair(ix, ox, X, Q, 10, probe=2, T=T, min_cand=tau)


def test_recursive_lattice_probing_large_k(e8pair):
    ix, ox, X, Q = e8pair
    run_query_pair(ix, ox, X, Q, 100, probe=2, T=256, min_cand=200)


def test_recursive_needs_one_table(blsh):
    cfg = synth.CONFIGS["c1"]
    X, Q = synth.make_dataset(cfg, n=3000, nq=16)
    ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=2, M=8, W=1.2, seed=3, quantizer=1, n_tables=2)
    with pytest.raises(blsh.BlshError):
        ix.query(torch.from_numpy(Q).cuda(), 10, probe=2, n_probes=256, min_cand=10)
    ix.close()
