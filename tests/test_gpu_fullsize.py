"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times.

c3 (configs[2], 1M x 384, 10k queries, k = 50, multiprobe T = 16 + Morton hierarchy
with the batch-median tau): the oracle builds the same index and answers the whole
batch (the median is a batch statistic), so the table is compared bit for bit, the
candidate counts of every query, and candidate sets + top-k on a sample.

c4 (configs[3], 10M x 384, 100k queries, k = 10, multiprobe T = 32; the bench
workload, in bench.py's launch configuration):
* against the oracle: the oracle builds the same 10M-point index (~2.5 min on the
  box's host cores) and the table (perm, bucket keys, offsets, leaf ranges) is
  compared bit for bit; 400 sampled queries go through the oracle's query phase and
  their leaf, codes, out-of-range flags, probe-key sequences, |A(q)|, candidate sets
  and top-k (check_topk) are compared with the GPU's answers to the whole batch;
* properties over the whole batch: the default (tensor-core screened) short-list
  equals the warp short-list bit for bit; reported distances are the exact fp64
  distances of the reported ids within 1e-5; lists are sorted and duplicate-free;
  recall@10 against the committed oracle brute-force ground truth on 1000 queries
  (bench_data/c4_gt.npz, tools/make_gt.py --sample 1000) is >= 0.9.
"""
import os

import numpy as np
import pytest

import synth
from parity_utils import TOL, check_topk, gpu_candidates

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def blsh():
    if not torch.cuda.is_available():
        pytest.skip("needs CUDA")
    from paper_conf_icde_panm12_b200 import blsh as b
    b.lib()
    return b


def test_c3_full_size_parity(blsh, orc):
    cfg = synth.CONFIGS["c3"]
    Xd, Qd = synth.make_dataset(cfg, backend="torch", device="cuda")
    X, Q = Xd.cpu().numpy(), Qd.cpu().numpy()
    ix = blsh.blsh_build(Xd, n_leaves=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index)
    ids, d2, nc = ix.query(Qd, cfg.k, probe=cfg.probe, n_probes=cfg.T, hierarchy=cfg.hierarchy,
                           min_cand=cfg.min_cand, keep_stages=True)
    torch.cuda.synchronize()
    ids, d2, nc = ids.cpu().numpy(), d2.cpu().numpy(), nc.cpu().numpy()
    ox = orc.OracleIndex(X, G=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index)
    for g, o in [("PERM", "perm"), ("UKEY", "ukey"), ("UOFF", "uoff"), ("LEAF_U", "leaf_u")]:
        assert np.array_equal(ix.export(g), ox.get(o).ravel()), f"{g} differs at full size"
    oi, od, onc = ox.query(Q, cfg.k, probe=cfg.probe, T=cfg.T, hierarchy=cfg.hierarchy, min_cand=cfg.min_cand)
    assert int(ix.export("Q_TAU")[0]) == ox.tau, "batch-median tau differs"
    assert np.array_equal(nc, onc), "|A(q)| differs"
    assert np.array_equal(ix.export("Q_LEVEL"), ox.get("q_level")), "hierarchy levels differ"
    rng = np.random.default_rng(3)
    sample = np.sort(rng.choice(len(Q), 300, replace=False))
    gc = gpu_candidates(ix, cfg.T)
    oc = ox.candidates()
    for q in sample:
        assert np.array_equal(gc[q], oc[q]), f"candidate set of query {q} differs"
    check_topk(ids[sample], d2[sample], oi[sample], od[sample], X, Q[sample], cands=[oc[q] for q in sample])


@pytest.fixture(scope="module")
def c4_gpu(blsh):
    cfg = synth.CONFIGS["c4"]
    Xd, Qd = synth.make_dataset(cfg, backend="torch", device="cuda")
    ix = blsh.blsh_build(Xd, n_leaves=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index, keep_stages=True)
    yield cfg, Xd, Qd, ix
    ix.close()


def test_c4_full_size_oracle_parity(c4_gpu, orc):
    cfg, Xd, Qd, ix = c4_gpu
    kw = dict(probe=cfg.probe, n_probes=cfg.T, hierarchy=cfg.hierarchy, min_cand=cfg.min_cand)
    ids, d2, nc = ix.query(Qd, cfg.k, keep_stages=True, **kw)
    torch.cuda.synchronize()
    assert ix.stats().tiled == 2, "the bench launch configuration runs the tensor-core short-list"
    ids, d2, nc = ids.cpu().numpy(), d2.cpu().numpy(), nc.cpu().numpy()
    T = cfg.T
    g_leaf, g_code, g_oor = ix.export("Q_LEAF"), ix.export("Q_CODE").reshape(-1, cfg.M), ix.export("Q_OOR")
    g_pkey = ix.export("Q_PKEY").reshape(cfg.nq, T, 2)
    g_pval = ix.export("Q_PVALID").reshape(cfg.nq, T)
    iv = ix.export("Q_INTERVALS").reshape(-1, T + 1, 2)
    perm = ix.export("PERM")
    X = Xd.cpu().numpy()
    ox = orc.OracleIndex(X, G=cfg.G, M=cfg.M, W=cfg.W, seed=cfg.seed_index)
    for g, o in [("PERM", "perm"), ("UKEY", "ukey"), ("UOFF", "uoff"), ("LEAF_U", "leaf_u")]:
        assert np.array_equal(ix.export(g), ox.get(o).ravel()), f"{g} differs at full size"
    rng = np.random.default_rng(44)
    sample = np.sort(rng.choice(cfg.nq, 400, replace=False))
    Qs = Qd[torch.as_tensor(sample, device="cuda")].cpu().numpy()
    oi, od, onc = ox.query(Qs, cfg.k, probe=cfg.probe, T=T, hierarchy=cfg.hierarchy, min_cand=cfg.min_cand)
    assert np.array_equal(g_leaf[sample], ox.get("q_leaf")), "query leaves differ"
    assert np.array_equal(g_code[sample].ravel(), ox.get("q_code").ravel()), "query codes differ"
    assert np.array_equal(g_oor[sample], ox.get("q_oor")), "out-of-range flags differ"
    assert np.array_equal(g_pval[sample].ravel(), ox.get("q_pvalid").ravel()), "probe validity differs"
    assert np.array_equal(g_pkey[sample].ravel(), ox.get("q_pkey").ravel()), "probe-key sequences differ"
    assert np.array_equal(nc[sample], onc), "|A(q)| differs"
    oc = ox.candidates()
    for r, q in enumerate(sample):
        parts = [perm[a:b] for a, b in iv[q] if b > a]
        gq = np.sort(np.concatenate(parts)) if parts else np.zeros(0, np.int64)
        assert np.array_equal(gq, oc[r]), f"candidate set of query {q} differs"
    check_topk(ids[sample], d2[sample], oi, od, X, Qs, cands=oc)
    ox.close()


def test_c4_full_size_properties(c4_gpu, monkeypatch):
    cfg, Xd, Qd, ix = c4_gpu
    kw = dict(probe=cfg.probe, n_probes=cfg.T, hierarchy=cfg.hierarchy, min_cand=cfg.min_cand)
    ids, d2, nc = ix.query(Qd, cfg.k, **kw)
    torch.cuda.synchronize()
    assert ix.stats().tiled == 2, "the bench launch configuration runs the tensor-core short-list"
    monkeypatch.setenv("BLSH_SHORTLIST", "warp")
    wi, wd, wn = ix.query(Qd, cfg.k, **kw)
    torch.cuda.synchronize()
    assert ix.stats().tiled == 0
    monkeypatch.delenv("BLSH_SHORTLIST")
    assert torch.equal(nc, wn), "candidate counts differ between short-list kernels"
    assert torch.equal(ids, wi), "ids differ between the TC and warp short-lists"
    assert torch.equal(d2.view(torch.int32), wd.view(torch.int32)), "d2 bits differ between short-lists"
    # sorted, duplicate-free, padding only when |A(q)| < k
    fin = torch.isfinite(d2)
    assert torch.all(d2[:, 1:] >= d2[:, :-1])            # padding (+inf) sorts last
    assert torch.equal(fin.sum(1), torch.clamp(nc, max=cfg.k))
    # exact distances of the reported ids (fp64) on a sample
    rng = np.random.default_rng(4)
    sample = torch.as_tensor(np.sort(rng.choice(cfg.nq, 500, replace=False)), device="cuda")
    si, sd = ids[sample], d2[sample].double()
    ok = si >= 0
    rows = Xd[si.clamp(min=0)].double()
    ex = ((rows - Qd[sample].double()[:, None, :]) ** 2).sum(-1)
    assert torch.all((ex - sd).abs()[ok] <= TOL * ex[ok] + 1e-30), "reported d2 is not the distance of the id"
    srt = torch.sort(si, dim=1).values
    assert torch.all((srt[:, 1:] != srt[:, :-1]) | (srt[:, 1:] < 0)), "duplicate ids"
    # recall@10 against the oracle's brute-force ground truth
    path = os.path.join(ROOT, "bench_data", "c4_gt.npz")
    g = np.load(path)
    qidx = torch.as_tensor(g["qidx"], device="cuda")
    fpx = float(Xd[:: max(1, cfg.n // 997)].double().sum())
    assert abs(fpx - float(g["fp_x"])) <= 1e-6 * max(1.0, abs(float(g["fp_x"]))), "ground truth for other data"
    got = ids[qidx][:, :10].cpu().numpy()
    kth = g["d2"][:, 9].astype(np.float64)
    assert len(got) >= 1000, "SURVEY D5: recall on a 1000-query oracle sample"
    hits = 0
    for r in range(len(got)):
        gs = set(g["ids"][r, :10].tolist())
        for i in got[r]:
            if i >= 0 and (int(i) in gs or float(((Xd[int(i)].double() - Qd[int(g["qidx"][r])].double()) ** 2).sum())
                           <= kth[r] * (1 + 1e-5)):
                hits += 1
    assert hits / (10.0 * len(got)) >= 0.9
