"""CPU oracle for FastPSO's hot path — TEST INFRASTRUCTURE ONLY.

Thin ctypes wrapper over ``oracle/liboracle.so`` (built from pso_oracle.cpp with
``-O3 -ffp-contract=off``).  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
module.  It shares no code with the CUDA product path
(``paper_conf_icpp_liuwc21_b200/``) and imports nothing from it.

Citations (P:Lnnn = /root/reference/PAPER.md line nnn): Alg. 1 P:L81-103,
Eq. 1/2 P:L105-115, Eq. 4, Eq. 5, Sec 3.1-3.3 P:L135-153,
objectives P:L287-305 and [20].  Readings: DESIGN.md.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")

SPHERE, RASTRIGIN, ROSENBROCK, GRIEWANK, ACKLEY, EASOM = 1, 2, 3, 4, 5, 6
TAG_R1, TAG_R2, TAG_X0, TAG_V0 = 0, 1, 2, 3


class _Params(C.Structure):
    _fields_ = [
        ("n", C.c_int64), ("d", C.c_int32), ("objective", C.c_int32),
        ("w", C.c_float), ("c1", C.c_float), ("c2", C.c_float),
        ("lo", C.c_float), ("hi", C.c_float), ("vmax", C.c_float),
        ("seed", C.c_uint64), ("bounds", C.c_void_p),
    ]


_fp = C.POINTER(C.c_float)


class _State(C.Structure):
    _fields_ = [
        ("row_begin", C.c_int64), ("nrows", C.c_int64),
        ("X", _fp), ("V", _fp), ("PB", _fp), ("pf", _fp), ("f", _fp), ("G", _fp),
        ("gf", C.c_float), ("gi", C.c_int64), ("t", C.c_uint64),
    ]


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"oracle not built: {LIB_PATH} (run `make oracle`)")
        L = C.CDLL(LIB_PATH)
        u32p = C.POINTER(C.c_uint32)
        L.orc_philox4x32_10.argtypes = [u32p, u32p, u32p]
        L.orc_word.argtypes = [C.c_uint64, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32]
        L.orc_word.restype = C.c_uint32
        L.orc_uniform.argtypes = [C.c_uint32]
        L.orc_uniform.restype = C.c_float
        L.orc_words.argtypes = [C.c_uint64, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32,
                                C.c_int64, u32p]
        L.orc_objective_f64.argtypes = [C.c_int32, _fp, C.c_int32]
        L.orc_objective_f64.restype = C.c_double
        L.orc_objective.argtypes = [C.c_int32, _fp, C.c_int32]
        L.orc_objective.restype = C.c_float
        L.orc_objective_rows.argtypes = [C.c_int32, _fp, C.c_int64, C.c_int32, _fp]
        L.orc_default_vmax.argtypes = [C.c_float, C.c_float]
        L.orc_default_vmax.restype = C.c_float
        SP, PP = C.POINTER(_State), C.POINTER(_Params)
        L.orc_init_local.argtypes = [PP, SP, _fp, C.POINTER(C.c_int64), _fp]
        L.orc_step_local.argtypes = [PP, SP, C.POINTER(C.c_int), _fp, C.POINTER(C.c_int64), _fp]
        L.orc_merge.argtypes = [SP, C.c_int32, C.c_int32, C.POINTER(C.c_int), _fp,
                                C.POINTER(C.c_int64), _fp, C.c_int]
        L.orc_create.argtypes = [PP, SP, C.c_int32]
        L.orc_step.argtypes = [PP, SP, C.c_int64, C.c_int32]
        L.orc_rebest.argtypes = [PP, SP]
        L.orc_rows_step.argtypes = [PP, C.c_uint64, _fp, C.POINTER(C.c_int64), C.c_int64,
                                    _fp, _fp, _fp, _fp, _fp]
        _lib = L
    return _lib


def _f(a: np.ndarray):
    assert a.dtype == np.float32 and a.flags.c_contiguous
    return a.ctypes.data_as(_fp)


# ---------------------------------------------------------------- primitives
def philox4x32_10(ctr, key) -> np.ndarray:
    c = (C.c_uint32 * 4)(*[int(v) & 0xFFFFFFFF for v in ctr])
    k = (C.c_uint32 * 2)(*[int(v) & 0xFFFFFFFF for v in key])
    o = (C.c_uint32 * 4)()
    lib().orc_philox4x32_10(c, k, o)
    return np.array(list(o), dtype=np.uint32)


def word(seed, tag, t, i, j) -> int:
    return int(lib().orc_word(seed, tag, t, i, j))


def words(seed, tag, t, i, j0, m) -> np.ndarray:
    out = np.empty(m, dtype=np.uint32)
    lib().orc_words(seed, tag, t, i, j0, m, out.ctypes.data_as(C.POINTER(C.c_uint32)))
    return out


def uniform(w) -> float:
    return float(np.float32(lib().orc_uniform(int(w) & 0xFFFFFFFF)))


def objective(obj: int, x) -> float:
    x = np.ascontiguousarray(x, dtype=np.float32)
    return float(np.float32(lib().orc_objective(obj, _f(x), x.size)))


def objective_f64(obj: int, x) -> float:
    x = np.ascontiguousarray(x, dtype=np.float32)
    return float(lib().orc_objective_f64(obj, _f(x), x.size))


def objective_rows(obj: int, X) -> np.ndarray:
    X = np.ascontiguousarray(X, dtype=np.float32)
    out = np.empty(X.shape[0], dtype=np.float32)
    lib().orc_objective_rows(obj, _f(X), X.shape[0], X.shape[1], _f(out))
    return out


def default_vmax(lo, hi) -> float:
    return float(np.float32(lib().orc_default_vmax(lo, hi)))


# ---------------------------------------------------------------- swarm
class OracleSwarm:
    """A whole swarm (or one shard of it: global rows [row_begin, row_begin+nrows)).

    State arrays are numpy float32, dense row-major (nrows x d).  ``nshards``
    runs the create/step as k virtual particle shards with the same merge the
    multi-GPU path uses; results must not depend on k.
    """

    def __init__(self, n, d, w, c1, c2, lo, hi, objective, seed, vmax=0.0,
                 nshards=1, row_begin=0, nrows=None, create=True, bounds=None):
        self.p = _Params()
        self.p.n, self.p.d, self.p.objective = int(n), int(d), int(objective)
        self.p.w, self.p.c1, self.p.c2 = w, c1, c2
        self.p.lo, self.p.hi = lo, hi
        self.p.vmax = vmax if vmax > 0 else default_vmax(lo, hi)
        self.p.seed = int(seed) & 0xFFFFFFFFFFFFFFFF
        # per-dimension [vlo | vhi | xlo | xhi] (NEXT-2); kept alive with the swarm
        self.bounds = None
        if bounds is not None:
            self.bounds = np.ascontiguousarray(bounds, dtype=np.float32).reshape(4 * int(d))
            self.p.bounds = self.bounds.ctypes.data
        self.n, self.d, self.nshards = int(n), int(d), int(nshards)
        nrows = self.n - row_begin if nrows is None else int(nrows)
        self.row_begin, self.nrows = int(row_begin), nrows
        self.X = np.zeros((nrows, d), np.float32)
        self.V = np.zeros((nrows, d), np.float32)
        self.PB = np.zeros((nrows, d), np.float32)
        self.pf = np.zeros(nrows, np.float32)
        self.f = np.zeros(nrows, np.float32)
        self.G = np.zeros(d, np.float32)
        self.s = _State()
        self.s.row_begin, self.s.nrows = self.row_begin, nrows
        self.s.X, self.s.V, self.s.PB = _f(self.X), _f(self.V), _f(self.PB)
        self.s.pf, self.s.f, self.s.G = _f(self.pf), _f(self.f), _f(self.G)
        self.s.gf, self.s.gi, self.s.t = np.inf, 0, 0
        if create:
            lib().orc_create(C.byref(self.p), C.byref(self.s), self.nshards)

    @property
    def vmax(self) -> float:
        return float(np.float32(self.p.vmax))

    @property
    def gf(self) -> float:
        return float(np.float32(self.s.gf))

    @property
    def gi(self) -> int:
        return int(self.s.gi)

    @property
    def t(self) -> int:
        return int(self.s.t)

    def step(self, iters=1):
        lib().orc_step(C.byref(self.p), C.byref(self.s), int(iters), self.nshards)
        return self

    # shard-level API (multi-process tests)
    def init_local(self):
        cf, ci, row = C.c_float(), C.c_int64(), np.zeros(self.d, np.float32)
        lib().orc_init_local(C.byref(self.p), C.byref(self.s), C.byref(cf), C.byref(ci), _f(row))
        return self.nrows > 0, float(np.float32(cf.value)), int(ci.value), row

    def step_local(self):
        has, cf, ci = C.c_int(), C.c_float(), C.c_int64()
        row = np.zeros(self.d, np.float32)
        lib().orc_step_local(C.byref(self.p), C.byref(self.s), C.byref(has), C.byref(cf),
                             C.byref(ci), _f(row))
        return bool(has.value), float(np.float32(cf.value)), int(ci.value), row

    def merge(self, has, cf, ci, rows, is_init):
        k = len(has)
        h = (C.c_int * k)(*[int(bool(v)) for v in has])
        f = np.ascontiguousarray(cf, dtype=np.float32)
        i = np.ascontiguousarray(ci, dtype=np.int64)
        r = np.ascontiguousarray(rows, dtype=np.float32).reshape(k, self.d)
        lib().orc_merge(C.byref(self.s), self.d, k, h, _f(f),
                        i.ctypes.data_as(C.POINTER(C.c_int64)), _f(r), int(bool(is_init)))

    def set_state(self, X, V, PB, pf, t=0):
        self.X[...] = X
        self.V[...] = V
        self.PB[...] = PB
        self.pf[...] = pf
        self.s.t = int(t)
        lib().orc_rebest(C.byref(self.p), C.byref(self.s))
        return self

    def rows_step(self, t, G, idx, X, V, PB, pf):
        """Move+eval+pbest for sampled rows (global indices idx) at iteration t."""
        idx = np.ascontiguousarray(idx, dtype=np.int64)
        X = np.array(X, dtype=np.float32, order="C", copy=True)
        V = np.array(V, dtype=np.float32, order="C", copy=True)
        PB = np.array(PB, dtype=np.float32, order="C", copy=True)
        pf = np.array(pf, dtype=np.float32, order="C", copy=True)
        G = np.ascontiguousarray(G, dtype=np.float32)
        f = np.zeros(idx.size, np.float32)
        lib().orc_rows_step(C.byref(self.p), int(t), _f(G),
                            idx.ctypes.data_as(C.POINTER(C.c_int64)), idx.size,
                            _f(X), _f(V), _f(PB), _f(pf), _f(f))
        return X, V, PB, pf, f
