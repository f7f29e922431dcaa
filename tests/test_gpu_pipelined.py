"""blsh_query_pipelined (include/blsh.h): a stream of host batches, uploads and downloads
overlapped with the search on the library's copy stream.  Every batch's answers must equal
a separate blsh_query call on it (bit for bit: ids, d2 bits, |A(q)|), including a batch-level
statistic (the hierarchy's median tau, R18, taken per batch), repeated pointers, and the
oracle for one batch (P:45 problem statement)."""
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


def _pinned(a):
    return torch.from_numpy(np.ascontiguousarray(a)).pin_memory()


@pytest.mark.parametrize("hier", [0, 1])
def test_pipelined_equals_separate_calls(blsh, hier):
    cfg = synth.CONFIGS["c1"]
    X, Q = synth.make_dataset(cfg, n=20000, nq=3000)
    ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=4, M=8, W=4.0, seed=5)
    kw = dict(probe=1, n_probes=8, hierarchy=hier)
    batches = [Q[0:1000], Q[1000:2000], Q[2000:3000], Q[0:1000]]   # the last repeats the first
    Qs = [_pinned(b) for b in batches]
    outs = ix.query_pipelined(Qs, 10, **kw)
    for b, (ids, d2, nc) in zip(batches, outs):
        ri, rd, rn = ix.query(b, 10, **kw)     # host arrays -> host answers
        assert np.array_equal(np.asarray(ids), ri)
        assert np.array_equal(np.asarray(d2).view(np.uint32), rd.view(np.uint32))
        assert np.array_equal(np.asarray(nc), rn)
    assert np.array_equal(np.asarray(outs[0][0]), np.asarray(outs[3][0]))
    ix.close()


def test_pipelined_repeated_pointers_and_oracle(blsh, orc):
    cfg = synth.CONFIGS["c1"]
    X, Q = synth.make_dataset(cfg, n=8000, nq=300)
    ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=4, M=8, W=4.0, seed=9)
    ox = orc.OracleIndex(X, G=4, M=8, W=4.0, seed=9)
    Qp = _pinned(Q)
    out = (torch.empty((300, 10), dtype=torch.int64).pin_memory(),
           torch.empty((300, 10), dtype=torch.float32).pin_memory(),
           torch.empty((300,), dtype=torch.int64).pin_memory())
    ix.query_pipelined([Qp] * 5, 10, probe=1, n_probes=16, outs=[out] * 5)
    oi, od, onc = ox.query(Q, 10, probe=1, T=16)
    assert np.array_equal(out[2].numpy(), onc), "candidate counts differ from the oracle"
    check_topk(out[0].numpy(), out[1].numpy(), oi, od, X, Q)
    ix.close()


def test_pipelined_rejects_device_buffers(blsh):
    cfg = synth.CONFIGS["c1"]
    X, Q = synth.make_dataset(cfg, n=2000, nq=64)
    ix = blsh.blsh_build(torch.from_numpy(X).cuda(), n_leaves=2, M=8, W=4.0, seed=1)
    with pytest.raises(blsh.BlshError):
        ix.query_pipelined([torch.from_numpy(Q).cuda()], 10)
    assert ix.query_pipelined([], 10) == []
    ix.close()
