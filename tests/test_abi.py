"""CPU-side checks of the C ABI library (no compute calls without a GPU)."""
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def blsh():
    from paper_conf_icde_panm12_b200 import build
    build.build()
    from paper_conf_icde_panm12_b200 import blsh as b
    b.lib()
    return b


def _declared():
    hdr = open(os.path.join(ROOT, "include", "blsh.h")).read()
    return sorted(set(re.findall(r"\b(blsh_[a-z_]+)\s*\(", hdr)))


def test_library_exports_every_declared_symbol(blsh):
    decl = _declared()
    assert "blsh_build" in decl and "blsh_query" in decl and "blsh_free" in decl
    out = subprocess.run(["nm", "-D", "--defined-only", blsh.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (blsh_\w+)", out))
    missing = [s for s in decl if s not in exported]
    assert not missing, f"not exported: {missing}"
    assert set(blsh.EXPORTED_SYMBOLS) == set(decl)


def test_library_is_sm100a(blsh):
    out = subprocess.run(["cuobjdump", "--list-elf", blsh.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_defaults_and_argument_errors_without_gpu(blsh):
    import ctypes as C
    p = blsh.BuildParams()
    blsh.lib().blsh_build_params_default(C.byref(p))
    assert (p.n_leaves, p.M, p.ek_iters, p.world) == (1, 8, 40, 1) and p.rp_mean_c == 10.0
    q = blsh.QueryParams()
    blsh.lib().blsh_query_params_default(C.byref(q))
    assert (q.probe, q.n_probes, q.hierarchy) == (0, 1, 0)
    X = np.zeros((10, 4), np.float32)
    for kw in (dict(n_leaves=3), dict(M=0), dict(M=7, quantizer=1), dict(W=-1.0), dict(n_leaves=4, world=3)):
        with pytest.raises(blsh.BlshError) as e:
            blsh.blsh_build(X, **kw)
        assert e.value.status == blsh.BLSH_ERR_INVALID
    # a valid request on a machine without a GPU fails loudly (no CPU fallback)
    import torch
    if not torch.cuda.is_available():
        with pytest.raises(blsh.BlshError) as e:
            blsh.blsh_build(X, n_leaves=2)
        assert e.value.status == blsh.BLSH_ERR_CUDA


def test_product_does_not_touch_oracle():
    pkg = os.path.join(ROOT, "paper_conf_icde_panm12_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".cpp", ".h")):
                src = open(os.path.join(dp, f)).read()
                assert "import oracle" not in src and "from oracle" not in src and "orc_" not in src, f
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c")):
            src = open(os.path.join(ROOT, "oracle", f)).read()
            assert "paper_conf_icde_panm12_b200" not in src.replace("paper_conf_icde_panm12_b200/", "") or f == "__init__.py"
