"""Thin Python binding of the C ABI in include/blsh.h (libblsh.so).

Argument marshalling only: every step of the build and of the query path runs
in the library's CUDA kernels.  Arrays may be torch tensors (CUDA or CPU) or
numpy arrays; CUDA tensors are passed as device pointers on the current torch
stream, host arrays as host pointers (the library stages them).  There is no
CPU fallback: if libblsh.so cannot be loaded, importing the functions raises.
"""
from __future__ import annotations

import ctypes as C
import os
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("BLSH_LIB_PATH") or os.path.join(_HERE, "_lib", "libblsh.so")   # (variant builds: experiments)

BLSH_OK, BLSH_ERR_INVALID, BLSH_ERR_OOM, BLSH_ERR_CUDA, BLSH_ERR_RANGE, BLSH_ERR_UNSUPPORTED = range(6)
_STATUS = {0: "OK", 1: "INVALID", 2: "OOM", 3: "CUDA", 4: "RANGE", 5: "UNSUPPORTED"}

EX = dict(A=0, B=1, W=2, DIRS=3, MU=4, THETA=5, NTYPE=6, DIAM2=7, DA2=8, PERM=10, UKEY=11, ULEAF=12,
          UOFF=13, LEAF_U=14, RGRP=15, GSTART=16, POINT_LEAF=20, POINT_CODE=21, POINT_KEY=22, Q_LEAF=30, Q_T=31, Q_CODE=32,
          Q_OOR=33, Q_KEY=34, Q_PKEY=35, Q_PVALID=36, Q_BASE=37, Q_LEVEL=38, Q_TAU=39, Q_INTERVALS=40,
          Q_CAND_OFF=41, Q_CAND=42)


class BuildParams(C.Structure):
    _fields_ = [("n_leaves", C.c_int32), ("rp_rule", C.c_int32), ("rp_mean_c", C.c_double),
                ("rp_max_jitter", C.c_double), ("ek_iters", C.c_int32), ("M", C.c_int32),
                ("quantizer", C.c_int32), ("W", C.c_float), ("W_leaf", C.c_void_p), ("seed", C.c_uint64),
                ("rank", C.c_int32), ("world", C.c_int32), ("stream", C.c_void_p),
                ("keep_stages", C.c_int32), ("n_tables", C.c_int32), ("leaf_split", C.c_void_p),
                ("W_rule", C.c_int32)]


class QueryParams(C.Structure):
    _fields_ = [("probe", C.c_int32), ("n_probes", C.c_int32), ("hierarchy", C.c_int32),
                ("hier_step_bits", C.c_int32), ("min_cand", C.c_int64), ("stream", C.c_void_p),
                ("keep_stages", C.c_int32), ("timing", C.c_int32), ("global_base", C.c_void_p),
                ("curve_perturb", C.c_int32), ("msb_min", C.c_int32)]


class Info(C.Structure):
    _fields_ = [("n", C.c_int64), ("n_owned", C.c_int64), ("nu", C.c_int64), ("d", C.c_int32),
                ("d_stride", C.c_int32), ("G", C.c_int32), ("M", C.c_int32), ("B", C.c_int32),
                ("quantizer", C.c_int32), ("leaf_lo", C.c_int32), ("leaf_hi", C.c_int32),
                ("device_bytes", C.c_int64), ("build_ms", C.c_double), ("n_tables", C.c_int32),
                ("pad_", C.c_int32)]


class Stats(C.Structure):
    _fields_ = [("nq", C.c_int64), ("n_active", C.c_int64), ("total_cand", C.c_int64),
                ("n_items", C.c_int64), ("tau", C.c_int64), ("chunk", C.c_int32),
                ("launches", C.c_int32), ("shortlist_bytes", C.c_double),
                ("ms_route_hash", C.c_float), ("ms_probe", C.c_float), ("ms_plan", C.c_float),
                ("ms_shortlist", C.c_float), ("ms_merge", C.c_float), ("ms_total", C.c_float),
                ("tiled", C.c_int32), ("pad_", C.c_int32), ("union_rows", C.c_int64),
                ("pairs_scored", C.c_int64), ("shortlist_flops", C.c_double),
                ("ms_screen", C.c_float), ("ms_rescore", C.c_float), ("union_bytes", C.c_double),
                ("pairs_kept", C.c_int64), ("k_slots", C.c_int64), ("screen_row_bytes", C.c_int32),
                ("screen_kind", C.c_int32)]


class BlshError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


_lib = None


def lib():
    """Load libblsh.so (build it with ``python -m paper_conf_icde_panm12_b200.build``)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"libblsh.so not found at {LIB_PATH}; run "
                              "`python -m paper_conf_icde_panm12_b200.build` (no CPU fallback exists)")
        L = C.CDLL(LIB_PATH)
        P, i32, i64 = C.c_void_p, C.c_int32, C.c_int64
        L.blsh_build_params_default.argtypes = [C.POINTER(BuildParams)]
        L.blsh_build_params_default.restype = None
        L.blsh_query_params_default.argtypes = [C.POINTER(QueryParams)]
        L.blsh_query_params_default.restype = None
        L.blsh_build.argtypes = [P, i64, i32, C.POINTER(BuildParams), C.POINTER(P)]
        L.blsh_build.restype = i32
        L.blsh_query.argtypes = [P, P, i64, i32, C.POINTER(QueryParams), P, P, P]
        L.blsh_query.restype = i32
        L.blsh_query_pipelined.argtypes = [P, i32, P, i64, i32, C.POINTER(QueryParams), P, P, P]
        L.blsh_query_pipelined.restype = i32
        L.blsh_query_packed.argtypes = [P, P, i64, i32, C.POINTER(QueryParams), P, P]
        L.blsh_query_packed.restype = i32
        L.blsh_query_base_counts.argtypes = [P, P, i64, C.POINTER(QueryParams), P]
        L.blsh_query_base_counts.restype = i32
        L.blsh_merge_topk.argtypes = [P, i32, i64, i32, P, P, P]
        L.blsh_merge_topk.restype = i32
        L.blsh_export.argtypes = [P, i32, P, C.c_size_t, C.POINTER(C.c_size_t)]
        L.blsh_export.restype = i32
        L.blsh_index_info.argtypes = [P, C.POINTER(Info)]
        L.blsh_index_info.restype = i32
        L.blsh_last_stats.argtypes = [P, C.POINTER(Stats)]
        L.blsh_last_stats.restype = i32
        L.blsh_free.argtypes = [P]
        L.blsh_free.restype = None
        L.blsh_last_error.argtypes = []
        L.blsh_last_error.restype = C.c_char_p
        _lib = L
    return _lib


EXPORTED_SYMBOLS = ("blsh_build_params_default", "blsh_query_params_default", "blsh_build", "blsh_query",
                    "blsh_query_pipelined",
                    "blsh_query_packed", "blsh_query_base_counts", "blsh_merge_topk", "blsh_export", "blsh_index_info",
                    "blsh_last_stats", "blsh_free", "blsh_last_error")


def blsh_last_error() -> str:
    return lib().blsh_last_error().decode()


def _check(st: int):
    if st != BLSH_OK:
        raise BlshError(st, blsh_last_error())


# --- array marshalling ----------------------------------------------------------

def _is_torch(a) -> bool:
    return type(a).__module__.startswith("torch")


def _ptr(a):
    """(pointer, keepalive, is_cuda) of a C-contiguous array."""
    if a is None:
        return None, None, False
    if _is_torch(a):
        if not a.is_contiguous():
            a = a.contiguous()
        return C.c_void_p(a.data_ptr()), a, a.is_cuda
    a = np.ascontiguousarray(a)
    return a.ctypes.data_as(C.c_void_p), a, False


def _stream_for(*arrays):
    for a in arrays:
        if a is not None and _is_torch(a) and a.is_cuda:
            import torch
            return C.c_void_p(torch.cuda.current_stream(a.device).cuda_stream)
    return C.c_void_p(0)


def _f32(a):
    if _is_torch(a):
        import torch
        return a.to(torch.float32).contiguous()
    return np.ascontiguousarray(a, dtype=np.float32)


# --- the ABI, same names ---------------------------------------------------------

def blsh_build(X, n_leaves: int = 1, M: int = 8, W: float = 4.0, seed: int = 42, quantizer: int = 0,
               rp_rule: int = 0, rp_mean_c: float = 10.0, rp_max_jitter: float = 0.0, ek_iters: int = 40,
               W_leaf=None, rank: int = 0, world: int = 1, keep_stages: bool = False,
               n_tables: int = 1, leaf_split=None, W_rule: int = 0) -> "Index":
    X = _f32(X)
    n, d = int(X.shape[0]), int(X.shape[1])
    p = BuildParams()
    lib().blsh_build_params_default(C.byref(p))
    p.n_leaves, p.M, p.W, p.seed, p.quantizer = n_leaves, M, W, seed, quantizer
    p.rp_rule, p.rp_mean_c, p.rp_max_jitter, p.ek_iters = rp_rule, rp_mean_c, rp_max_jitter, ek_iters
    p.rank, p.world, p.keep_stages = rank, world, int(bool(keep_stages))
    p.n_tables = n_tables
    p.W_rule = W_rule
    ls = None
    if leaf_split is not None:   # load-aware contiguous leaf -> rank assignment [world+1]
        ls = np.ascontiguousarray(np.asarray(leaf_split, dtype=np.int32))
        if ls.shape != (world + 1,):
            raise ValueError("leaf_split needs world + 1 entries")
        p.leaf_split = ls.ctypes.data_as(C.c_void_p)
    wl = None
    if W_leaf is not None:
        wl = np.ascontiguousarray(np.asarray(W_leaf, dtype=np.float32))
        p.W_leaf = wl.ctypes.data_as(C.c_void_p)
    xp, keep, _ = _ptr(X)
    p.stream = _stream_for(X)
    h = C.c_void_p()
    _check(lib().blsh_build(xp, n, d, C.byref(p), C.byref(h)))
    return Index(h, n, d, M)


def _qparams(probe, n_probes, hierarchy, hier_step_bits, min_cand, keep_stages, timing, stream, global_base=None,
             curve_perturb=0, msb_min=0):
    p = QueryParams()
    lib().blsh_query_params_default(C.byref(p))
    p.curve_perturb, p.msb_min = curve_perturb, msb_min
    p.probe, p.n_probes, p.hierarchy, p.hier_step_bits = probe, n_probes, int(hierarchy), hier_step_bits
    p.min_cand, p.keep_stages, p.timing, p.stream = min_cand, int(bool(keep_stages)), int(bool(timing)), stream
    if global_base is not None:
        p.global_base = C.c_void_p(global_base.data_ptr())   # CUDA int64 tensor [nq]
    return p


def _alloc_like(Q, shape, kind):
    if _is_torch(Q) and Q.is_cuda:
        import torch
        dt = {"i64": torch.int64, "f32": torch.float32, "u64": torch.int64}[kind]
        return torch.empty(shape, dtype=dt, device=Q.device)
    dt = {"i64": np.int64, "f32": np.float32, "u64": np.uint64}[kind]
    return np.empty(shape, dtype=dt)


def blsh_query(index: "Index", Q, k: int, probe: int = 0, n_probes: int = 1, hierarchy: int = 0,
               hier_step_bits: int = 0, min_cand: int = 0, keep_stages: bool = False, timing: bool = False,
               out=None, global_base=None, curve_perturb: int = 0, msb_min: int = 0):
    """-> (ids [nq,k] int64, dist2 [nq,k] fp32, ncand [nq] int64), on Q's device."""
    Q = _f32(Q)
    nq = int(Q.shape[0])
    if out is None:
        out = (_alloc_like(Q, (nq, k), "i64"), _alloc_like(Q, (nq, k), "f32"), _alloc_like(Q, (nq,), "i64"))
    ids, d2, nc = out
    p = _qparams(probe, n_probes, hierarchy, hier_step_bits, min_cand, keep_stages, timing, _stream_for(Q, ids),
                 global_base, curve_perturb, msb_min)
    qp, kq, _ = _ptr(Q)
    ip, ki, _ = _ptr(ids)
    dp, kd, _ = _ptr(d2)
    np_, kn, _ = _ptr(nc)
    _check(lib().blsh_query(index.handle, qp, nq, k, C.byref(p), ip, dp, np_))
    return ids, d2, nc


def blsh_query_pipelined(index: "Index", Qs, k: int, probe: int = 0, n_probes: int = 1, hierarchy: int = 0,
                         hier_step_bits: int = 0, min_cand: int = 0, timing: bool = False, outs=None,
                         global_base=None, curve_perturb: int = 0, msb_min: int = 0):
    """Qs: a list of HOST batches [nq, d] (equal nq; entries may repeat).  -> list of
    (ids, dist2, ncand) host arrays, one per batch (``outs`` supplies them; entries may repeat)."""
    Qs = [_f32(Q) for Q in Qs]
    nb = len(Qs)
    if nb == 0:
        return []
    nq = int(Qs[0].shape[0])
    if any(int(Q.shape[0]) != nq for Q in Qs):
        raise ValueError("every batch must have the same number of queries")
    if outs is None:
        outs = [(_alloc_like(Q, (nq, k), "i64"), _alloc_like(Q, (nq, k), "f32"), _alloc_like(Q, (nq,), "i64"))
                for Q in Qs]
    p = _qparams(probe, n_probes, hierarchy, hier_step_bits, min_cand, False, timing, C.c_void_p(0),
                 global_base, curve_perturb, msb_min)
    keep = []

    def arr(items):
        ptrs = []
        for a in items:
            ptr, ka, _ = _ptr(a)
            keep.append(ka)
            ptrs.append(ptr.value if ptr is not None else None)
        return (C.c_void_p * nb)(*ptrs)

    qa = arr(Qs)
    ia = arr([o[0] for o in outs])
    da = arr([o[1] for o in outs])
    na = arr([o[2] for o in outs])
    _check(lib().blsh_query_pipelined(index.handle, nb, qa, nq, k, C.byref(p), ia, da, na))
    return outs


def blsh_query_packed(index: "Index", Q, k: int, probe: int = 0, n_probes: int = 1, hierarchy: int = 0,
                      hier_step_bits: int = 0, min_cand: int = 0, timing: bool = False, out=None,
                      global_base=None, curve_perturb: int = 0, msb_min: int = 0):
    """-> (packed [nq,k] (uint64 bits; int64 for torch), ncand [nq])."""
    Q = _f32(Q)
    nq = int(Q.shape[0])
    if out is None:
        out = (_alloc_like(Q, (nq, k), "u64"), _alloc_like(Q, (nq,), "i64"))
    pk, nc = out
    p = _qparams(probe, n_probes, hierarchy, hier_step_bits, min_cand, False, timing, _stream_for(Q, pk),
                 global_base, curve_perturb, msb_min)
    qp, kq, _ = _ptr(Q)
    pp, kp, _ = _ptr(pk)
    np_, kn, _ = _ptr(nc)
    _check(lib().blsh_query_packed(index.handle, qp, nq, k, C.byref(p), pp, np_))
    return pk, nc


def blsh_query_base_counts(index: "Index", Q, probe: int = 0, n_probes: int = 1, timing: bool = False,
                           out=None, curve_perturb: int = 0, **_ignored):
    """a1-a4 only: |A0(q)| [nq] int64 (0 for queries another shard owns), on Q's device."""
    Q = _f32(Q)
    nq = int(Q.shape[0])
    if out is None:
        out = _alloc_like(Q, (nq,), "i64")
    p = _qparams(probe, n_probes, 0, 0, 0, False, timing, _stream_for(Q, out), None, curve_perturb)
    qp, kq, _ = _ptr(Q)
    op, ko, _ = _ptr(out)
    _check(lib().blsh_query_base_counts(index.handle, qp, nq, C.byref(p), op))
    return out


def blsh_merge_topk(packed, n_lists: int, nq: int, k: int, out=None):
    """packed: CUDA tensor [n_lists*nq*k] (int64 bits of the packed u64 entries)."""
    if out is None:
        out = (_alloc_like(packed, (nq, k), "i64"), _alloc_like(packed, (nq, k), "f32"))
    ids, d2 = out
    pp, kp, _ = _ptr(packed)
    ip, ki, _ = _ptr(ids)
    dp, kd, _ = _ptr(d2)
    _check(lib().blsh_merge_topk(pp, n_lists, nq, k, ip, dp, _stream_for(packed)))
    return ids, d2


_EX_DT = {"A": np.float32, "B": np.float32, "W": np.float32, "DIRS": np.float32, "MU": np.float32,
          "THETA": np.float32, "NTYPE": np.int32, "DIAM2": np.float64, "DA2": np.float64, "PERM": np.int64,
          "UKEY": np.uint64, "ULEAF": np.int32, "UOFF": np.int64, "LEAF_U": np.int64,
          "RGRP": np.int32, "GSTART": np.int64, "POINT_LEAF": np.int32,
          "POINT_CODE": np.int32, "POINT_KEY": np.uint64, "Q_LEAF": np.int32, "Q_T": np.float32,
          "Q_CODE": np.int32, "Q_OOR": np.int32, "Q_KEY": np.uint64, "Q_PKEY": np.uint64,
          "Q_PVALID": np.int32, "Q_BASE": np.int64, "Q_LEVEL": np.int32, "Q_TAU": np.int64,
          "Q_INTERVALS": np.int64, "Q_CAND_OFF": np.int64, "Q_CAND": np.int64}


def blsh_export(index: "Index", what: str, table: int = 0) -> np.ndarray:
    """Host copy of a build artefact / last-query stage; ``table`` selects hash
    table l of an L-table index for the per-table items (BLSH_EX_TABLE)."""
    code = EX[what] | (int(table) << 8)
    need = C.c_size_t(0)
    lib().blsh_export(index.handle, code, None, 0, C.byref(need))
    dt = _EX_DT[what]
    out = np.zeros(max(need.value // np.dtype(dt).itemsize, 0), dtype=dt)
    if need.value:
        _check(lib().blsh_export(index.handle, code, out.ctypes.data_as(C.c_void_p), need.value, None))
    return out


def blsh_index_info(index: "Index") -> Info:
    i = Info()
    _check(lib().blsh_index_info(index.handle, C.byref(i)))
    return i


def blsh_last_stats(index: "Index") -> Stats:
    s = Stats()
    _check(lib().blsh_last_stats(index.handle, C.byref(s)))
    return s


def blsh_free(index: "Index") -> None:
    if index.handle:
        lib().blsh_free(index.handle)
        index.handle = None


class Index:
    """Owning handle of a blsh_index (frees on close / garbage collection)."""

    def __init__(self, handle, n, d, M):
        self.handle = handle
        self.n, self.d, self.M = n, d, M

    def query(self, Q, k, **kw):
        return blsh_query(self, Q, k, **kw)

    def query_pipelined(self, Qs, k, **kw):
        return blsh_query_pipelined(self, Qs, k, **kw)

    def query_packed(self, Q, k, **kw):
        return blsh_query_packed(self, Q, k, **kw)

    def base_counts(self, Q, **kw):
        return blsh_query_base_counts(self, Q, **kw)

    def export(self, what: str, table: int = 0) -> np.ndarray:
        return blsh_export(self, what, table)

    def info(self) -> Info:
        return blsh_index_info(self)

    def stats(self) -> Stats:
        return blsh_last_stats(self)

    def close(self):
        blsh_free(self)

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
