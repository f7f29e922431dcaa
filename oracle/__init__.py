"""CPU oracle for Bi-level LSH -- TEST INFRASTRUCTURE ONLY.

ctypes wrapper around ``oracle/liboracle.so`` (plain C, ``blsh_oracle.c``).
Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  It
shares no code with ``paper_conf_icde_panm12_b200`` (the CUDA product) and
never imports it.  See DESIGN.md "Oracle" for what each function follows.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "blsh_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

CFLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fopenmp", "-shared",
          "-fPIC"]


def build(force: bool = False) -> str:
    """Compile liboracle.so (gcc; no fast-math, no fp contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB)
        P = C.c_void_p
        i64, i32, u64, f32, f64 = C.c_int64, C.c_int, C.c_uint64, C.c_float, C.c_double
        L.orc_rng_u64.restype = u64
        L.orc_rng_u64.argtypes = [u64, u64, u64]
        L.orc_rng_uniform.restype = f64
        L.orc_rng_uniform.argtypes = [u64, u64, u64]
        L.orc_rng_gauss.restype = f64
        L.orc_rng_gauss.argtypes = [u64, u64, u64]
        L.orc_gen_params.restype = None
        L.orc_gen_params.argtypes = [u64, i32, i32, i32, P, P, P, P, P]
        L.orc_dot_canonical.restype = f32
        L.orc_dot_canonical.argtypes = [P, P, i32]
        L.orc_dist2_canonical.restype = f32
        L.orc_dist2_canonical.argtypes = [P, P, i32]
        L.orc_bits_per_coord.restype = i32
        L.orc_bits_per_coord.argtypes = [i32]
        L.orc_morton_encode.restype = None
        L.orc_morton_encode.argtypes = [P, i32, P, P]
        L.orc_morton_decode.restype = None
        L.orc_morton_decode.argtypes = [u64, u64, i32, P]
        L.orc_e8_decode.restype = None
        L.orc_e8_decode.argtypes = [P, P]
        L.orc_e8_roots.restype = None
        L.orc_e8_roots.argtypes = [P]
        L.orc_multiprobe_deltas.restype = i32
        L.orc_multiprobe_deltas.argtypes = [P, i32, i32, P, P]
        L.orc_lattice_order.restype = i32
        L.orc_lattice_order.argtypes = [P, P, i32, P]
        L.orc_hash_point.restype = None
        L.orc_hash_point.argtypes = [P, P, f32, i32, i32, P, P, P]
        L.orc_diameter_estimate.restype = f32
        L.orc_diameter_estimate.argtypes = [P, i32, P, i64, i32, P, P]
        L.orc_build.restype = P
        L.orc_build.argtypes = [P, i64, i32, i32, i32, i32, f32, P, i32, f64, f64, i32, u64, i32, i32,
                                C.POINTER(C.c_int)]
        L.orc_free.restype = None
        L.orc_free.argtypes = [P]
        L.orc_query.restype = i32
        L.orc_query.argtypes = [P, P, i64, i32, i32, i32, i32, i32, i64, P, P, P]
        L.orc_e8_second_ring.restype = i32
        L.orc_e8_second_ring.argtypes = [P]
        L.orc_e8_parent.restype = None
        L.orc_e8_parent.argtypes = [P, P]
        L.orc_query_ex.restype = i32
        L.orc_query_ex.argtypes = [P, P, i64, i32, i32, i32, i32, i32, i64, i32, i32, P, P, P]
        L.orc_query_union.restype = i32
        L.orc_query_union.argtypes = [P, i32, P, i64, i32, i32, i32, P, P, P]
        L.orc_gen_table_params.restype = None
        L.orc_gen_table_params.argtypes = [u64, i32, i32, i32, i32, P, P, P]
        L.orc_bruteforce.restype = None
        L.orc_bruteforce.argtypes = [P, i64, i32, P, i64, i32, P, P]
        L.orc_info.restype = None
        L.orc_info.argtypes = [P, P]
        L.orc_last_ncand_total.restype = i64
        L.orc_last_ncand_total.argtypes = [P]
        L.orc_get.restype = i32
        L.orc_get.argtypes = [P, i32, P]
        L.orc_num_threads.restype = i32
        L.orc_num_threads.argtypes = []
        L.orc_set_num_threads.restype = None
        L.orc_set_num_threads.argtypes = [i32]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


def _f32(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.float32)


# --- primitives --------------------------------------------------------------

def rng_u64(seed: int, stream: int, i: int) -> int:
    return int(lib().orc_rng_u64(seed, stream, i))


def rng_uniform(seed: int, stream: int, i: int) -> float:
    return float(lib().orc_rng_uniform(seed, stream, i))


def rng_gauss(seed: int, stream: int, i: int) -> float:
    return float(lib().orc_rng_gauss(seed, stream, i))


def gen_params(seed: int, G: int, M: int, d: int, W):
    """(A [G,M,d], b [G,M], dirs [G-1,d], jit [G-1]) per reading R2."""
    Wl = _f32(np.broadcast_to(np.asarray(W, dtype=np.float32), (G,)))
    A = np.empty((G, M, d), np.float32)
    b = np.empty((G, M), np.float32)
    dirs = np.zeros((max(G - 1, 1), d), np.float32)
    jit = np.zeros(max(G - 1, 1), np.float64)
    lib().orc_gen_params(seed, G, M, d, _p(Wl), _p(A), _p(b), _p(dirs), _p(jit))
    return A, b, dirs[:G - 1], jit[:G - 1]


def gen_table_params(seed: int, table: int, G: int, M: int, d: int, W):
    """(A [G,M,d], b [G,M]) of hash table ``table`` (P:43 L tables, R2/R24)."""
    Wl = _f32(np.broadcast_to(np.asarray(W, dtype=np.float32), (G,)))
    A = np.empty((G, M, d), np.float32)
    b = np.empty((G, M), np.float32)
    lib().orc_gen_table_params(seed, table, G, M, d, _p(Wl), _p(A), _p(b))
    return A, b


def dot_canonical(a, x) -> np.float32:
    a, x = _f32(a), _f32(x)
    return np.float32(lib().orc_dot_canonical(_p(a), _p(x), a.size))


def dist2_canonical(x, y) -> np.float32:
    x, y = _f32(x), _f32(y)
    return np.float32(lib().orc_dist2_canonical(_p(x), _p(y), x.size))


def hash_point(A, b, W: float, x):
    """Eq. 2 with explicit parameters: (t [M] fp32, h [M] int32)."""
    A, b, x = _f32(A), _f32(b), _f32(x)
    M, d = A.shape
    t = np.empty(M, np.float32)
    h = np.empty(M, np.int32)
    lib().orc_hash_point(_p(A), _p(b), float(W), M, d, _p(x), _p(t), _p(h))
    return t, h


def bits_per_coord(M: int) -> int:
    return int(lib().orc_bits_per_coord(M))


def morton_encode(code) -> int:
    c = np.ascontiguousarray(code, dtype=np.int32)
    hi, lo = C.c_uint64(), C.c_uint64()
    lib().orc_morton_encode(_p(c), c.size, C.byref(hi), C.byref(lo))
    return (hi.value << 64) | lo.value


def morton_decode(key: int, M: int) -> np.ndarray:
    out = np.empty(M, np.int32)
    lib().orc_morton_decode((key >> 64) & (2**64 - 1), key & (2**64 - 1), M, _p(out))
    return out


def e8_decode(y) -> np.ndarray:
    """Nearest E8 point of y (8 floats), returned in doubled coordinates (2c)."""
    y = _f32(y)
    out = np.empty(8, np.int32)
    lib().orc_e8_decode(_p(y), _p(out))
    return out


def e8_second_ring() -> np.ndarray:
    """The 9120 second-ring E8 vectors of recursive probing (R26), doubled coordinates, canonical order."""
    out = np.zeros((9120, 8), np.int32)
    n = lib().orc_e8_second_ring(_p(out))
    assert n == 9120, n
    return out


def e8_parent(c2) -> np.ndarray:
    """Parent code in the E8 hierarchy (Eq. 10, R27), doubled coordinates: DECODE(c2 / 4)."""
    c = np.ascontiguousarray(c2, dtype=np.int32)
    out = np.empty(8, np.int32)
    lib().orc_e8_parent(_p(c), _p(out))
    return out


def e8_roots() -> np.ndarray:
    out = np.empty((240, 8), np.int32)
    lib().orc_e8_roots(_p(out))
    return out


def multiprobe_deltas(t, T: int):
    t = _f32(t)
    M = t.size
    deltas = np.zeros((max(T - 1, 1), M), np.int32)
    scores = np.zeros(max(T - 1, 1), np.float64)
    rc = lib().orc_multiprobe_deltas(_p(t), M, T, _p(deltas), _p(scores))
    if rc != 0:
        raise ValueError("multiprobe_deltas: invalid arguments")
    return deltas[:T - 1], scores[:T - 1]


def lattice_order(y, c2, T: int) -> np.ndarray:
    y = _f32(y)
    c2 = np.ascontiguousarray(c2, dtype=np.int32)
    out = np.zeros(max(T - 1, 1), np.int32)
    rc = lib().orc_lattice_order(_p(y), _p(c2), T, _p(out))
    if rc != 0:
        raise ValueError("lattice_order: invalid arguments")
    return out[:T - 1]


def diameter_estimate(X, ids, m: int = 40):
    """(est^2, r1^2, selected ids) of reading R6 over the rows ``ids`` of X."""
    X = _f32(X)
    ids = np.ascontiguousarray(ids, dtype=np.int64)
    r1 = C.c_float()
    mm = min(m, ids.size) if ids.size else 1
    sel = np.zeros(max(mm, 1), np.int64)
    v = lib().orc_diameter_estimate(_p(X), X.shape[1], _p(ids), ids.size, m, C.byref(r1), _p(sel))
    return float(v), float(r1.value), sel[:mm]


def bruteforce(X, Q, k: int):
    """Exact k-NN in fp64 (ids, dist2 as fp32), ties by id."""
    X, Q = _f32(X), _f32(Q)
    nq = Q.shape[0]
    ids = np.empty((nq, k), np.int64)
    d2 = np.empty((nq, k), np.float32)
    lib().orc_bruteforce(_p(X), X.shape[0], X.shape[1], _p(Q), nq, k, _p(ids), _p(d2))
    return ids, d2


def num_threads() -> int:
    return int(lib().orc_num_threads())


def set_num_threads(n: int) -> None:
    lib().orc_set_num_threads(int(n))


# --- index -------------------------------------------------------------------

class OracleError(RuntimeError):
    pass


class OracleIndex:
    """Plain Bi-level LSH index built by the oracle (b1-b4 of SURVEY §8(a))."""

    _GET = {
        "A": (0, np.float32, lambda s: (s.G, s.M, s.d)),
        "b": (1, np.float32, lambda s: (s.G, s.M)),
        "dirs": (2, np.float32, lambda s: (max(s.G - 1, 0), s.d)),
        "theta": (3, np.float32, lambda s: (max(s.G - 1, 0),)),
        "ntype": (4, np.int32, lambda s: (max(s.G - 1, 0),)),
        "mu": (5, np.float32, lambda s: (max(s.G - 1, 0), s.d)),
        "leaf": (6, np.int32, lambda s: (s.n,)),
        "code": (7, np.int32, lambda s: (s.n, s.M)),
        "key": (8, np.uint64, lambda s: (s.n, 2)),
        "perm": (9, np.int64, lambda s: (s.n,)),
        "ukey": (10, np.uint64, lambda s: (s.nu, 2)),
        "uleaf": (11, np.int32, lambda s: (s.nu,)),
        "uoff": (12, np.int64, lambda s: (s.nu + 1,)),
        "leaf_u": (13, np.int64, lambda s: (s.G + 1,)),
        "W": (14, np.float32, lambda s: (s.G,)),
        "diam2": (15, np.float64, lambda s: (max(s.G - 1, 0),)),
        "da2": (16, np.float64, lambda s: (max(s.G - 1, 0),)),
        "jit": (17, np.float64, lambda s: (max(s.G - 1, 0),)),
        "q_leaf": (20, np.int32, lambda s: (s.lq_n,)),
        "q_t": (21, np.float32, lambda s: (s.lq_n, s.M)),
        "q_code": (22, np.int32, lambda s: (s.lq_n, s.M)),
        "q_oor": (23, np.int32, lambda s: (s.lq_n,)),
        "q_key": (24, np.uint64, lambda s: (s.lq_n, 2)),
        "q_pkey": (25, np.uint64, lambda s: (s.lq_n, s.lq_T, 2)),
        "q_pvalid": (26, np.int32, lambda s: (s.lq_n, s.lq_T)),
        "q_base": (27, np.int64, lambda s: (s.lq_n,)),
        "q_level": (28, np.int32, lambda s: (s.lq_n,)),
        "q_coff": (29, np.int64, lambda s: (s.lq_n + 1,)),
        "q_cand": (30, np.int64, lambda s: (s.ncand_total,)),
    }

    def __init__(self, X, G: int, M: int = 8, W: float = 4.0, seed: int = 42, quantizer: int = 0,
                 W_leaf=None, rp_rule: int = 0, rp_mean_c: float = 10.0,
                 rp_max_jitter: float = 0.0, ek_iters: int = 40, L: int = 1, W_rule: int = 0):
        """L > 1: L independent hash tables over the same RP-tree; table l
        is the single-table index built with table = l (its own (a, b))."""
        self.X = _f32(X)
        n, d = self.X.shape
        Wl = None if W_leaf is None else _f32(W_leaf)
        self._tabs = []
        for l in range(L):
            err = C.c_int(0)
            h = lib().orc_build(_p(self.X), n, d, G, M, quantizer, float(W),
                                _p(Wl) if Wl is not None else None, rp_rule, float(rp_mean_c),
                                float(rp_max_jitter), ek_iters, seed, l, W_rule, C.byref(err))
            if not h:
                self.close()
                raise OracleError(f"orc_build failed (code {err.value})", err.value)
            self._tabs.append(h)
        self._h = self._tabs[0]
        self._Wl = Wl
        self.L = L
        self.n, self.d, self.G, self.M = n, d, G, M
        self.quantizer = quantizer
        self.lq_T = 1
        self._refresh()

    def _refresh(self, table: int = 0):
        info = np.zeros(8, np.int64)
        h = self._tabs[table]
        lib().orc_info(h, _p(info))
        self.B = int(info[4])
        self.nu = int(info[5])
        self.lq_n = int(info[6])
        self.tau = int(info[7])
        self.ncand_total = int(lib().orc_last_ncand_total(h))

    def get(self, what: str, table: int = 0) -> np.ndarray:
        code, dt, shape = self._GET[what]
        self._refresh(table)
        out = np.zeros(shape(self), dt)
        if out.size:
            rc = lib().orc_get(self._tabs[table], code, _p(out))
            if rc:
                raise OracleError(f"orc_get({what}) failed")
        self._refresh(0)
        return out

    def query(self, Q, k: int, probe: int = 0, T: int = 1, hierarchy: int = 0,
              hier_step_bits: int = 0, min_cand: int = 0, curve_perturb: int = 0, msb_min: int = 0):
        Q = _f32(Q)
        nq = Q.shape[0]
        ids = np.empty((nq, k), np.int64)
        d2 = np.empty((nq, k), np.float32)
        nc = np.empty(nq, np.int64)
        if self.L == 1:
            rc = lib().orc_query_ex(self._h, _p(Q), nq, k, probe, T, hierarchy, hier_step_bits,
                                    min_cand, curve_perturb, msb_min, _p(ids), _p(d2), _p(nc))
        elif hierarchy:
            raise OracleError("the Morton hierarchy is defined for L = 1 only (R24)")
        else:
            arr = (C.c_void_p * self.L)(*self._tabs)
            rc = lib().orc_query_union(arr, self.L, _p(Q), nq, k, probe, T, _p(ids), _p(d2), _p(nc))
        if rc:
            raise OracleError("orc_query: invalid arguments")
        self.lq_T = T
        self._refresh()
        return ids, d2, nc

    def candidates(self, table=None):
        """Candidate id sets A(q) of the last query (sorted arrays): the union
        over the L tables, or one table's set when ``table`` is given."""
        tabs = range(self.L) if table is None else [table]
        per = []
        for l in tabs:
            off = self.get("q_coff", l)
            ids = self.get("q_cand", l)
            per.append([ids[off[i]:off[i + 1]] for i in range(len(off) - 1)])
        if len(per) == 1:
            return per[0]
        return [np.unique(np.concatenate([p[q] for p in per])) for q in range(len(per[0]))]

    def close(self):
        for h in getattr(self, "_tabs", []):
            if h:
                lib().orc_free(h)
        self._tabs = []
        self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
