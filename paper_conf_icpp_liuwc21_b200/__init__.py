"""B200-native FastPSO hot path (Liu, Wen, Cai — ICPP'21).

Python surface over the C ABI in include/fastpso.h.  Marshalling only: the
swarm lives in device memory owned by the CUDA library; each ``step`` runs one
fused sm_100a kernel per PSO iteration.  Host buffers may be
numpy arrays or CPU torch tensors (pinned or not); they are passed by pointer.
"""
from __future__ import annotations

import ctypes as C

import numpy as np

from ._lib import (EXPORTS, PSO_D_AUTO_COLSPLIT, PSO_D_MAX, PSO_D_MAX_ROW, PSO_FLAG_ASYNC_GBEST,
                   PSO_FLAG_ALLREDUCE, PSO_FLAG_COLUMN_SPLIT, PSO_FLAG_DEFER_INIT, PSO_FLAG_DEVICE, PSO_FLAG_TIMING, PSO_OBJ_ACKLEY, PSO_OBJ_CUSTOM_BASE,
                   PSO_OBJ_EASOM, PSO_OBJ_GRIEWANK, PSO_OBJ_RASTRIGIN, PSO_OBJ_ROSENBROCK,
                   PSO_OBJ_SPHERE, PSO_OK, PsoError, check, last_error, lib, pso_info, pso_opts,
                   status_string)

__all__ = [
    "Swarm", "PsoError", "lib", "check", "status_string", "last_error", "objective_registered",
    "debug_philox", "debug_objective", "nccl_unique_id", "nccl_comm_init", "nccl_comm_destroy",
    "PSO_OBJ_SPHERE", "PSO_OBJ_RASTRIGIN", "PSO_OBJ_ROSENBROCK", "PSO_OBJ_GRIEWANK",
    "PSO_OBJ_ACKLEY", "PSO_OBJ_EASOM", "PSO_OBJ_CUSTOM_BASE", "PSO_FLAG_TIMING", "PSO_D_MAX",
    "PSO_D_MAX_ROW", "PSO_D_AUTO_COLSPLIT",
    "EXPORTS",
]


def _ptr(a, count=None, writable=False, dtype=np.float32):
    """Raw host pointer of a C-contiguous numpy array or CPU torch tensor (or None).

    The library reads or writes exactly ``count`` elements of ``dtype`` behind
    the pointer, so both the element type and the element count are checked
    here (a float16 or undersized output would be a host heap overflow, a
    float64 input would be silently reinterpreted)."""
    if a is None:
        return None
    if hasattr(a, "data_ptr"):  # torch.Tensor
        import torch
        want = {np.dtype(np.float32): torch.float32}[np.dtype(dtype)]
        if a.device.type != "cpu" or not a.is_contiguous():
            raise ValueError("host tensors must be contiguous CPU tensors")
        if a.dtype != want:
            raise ValueError(f"expected a {want} tensor, got {a.dtype}")
        size = a.numel()
        ptr = a.data_ptr()
    else:
        if not isinstance(a, np.ndarray) or a.dtype != dtype or not a.flags.c_contiguous:
            raise ValueError(f"expected a C-contiguous numpy {np.dtype(dtype).name} array")
        if writable and not a.flags.writeable:
            raise ValueError("output array is read-only")
        size = a.size
        ptr = a.ctypes.data
    if count is not None and size != count:
        raise ValueError(f"buffer holds {size} elements, the call needs exactly {count}")
    return C.c_void_p(ptr)


def objective_registered(obj: int) -> bool:
    return bool(lib().pso_objective_registered(int(obj)))


class Swarm:
    """One handle of the C ABI (pso_create_ex ... pso_destroy)."""

    def __init__(self, n: int, d: int, w: float, c1: float, c2: float, lo: float, hi: float,
                 objective: int, seed: int, *, vmax: float = 0.0, device: int = -1,
                 stream=None, nccl_comm=None, timing: bool = False, bounds=None,
                 world: int = 1, rank: int = 0, defer_init: bool = False,
                 async_gbest: bool = False, column_split: bool = False,
                 allreduce_exchange: bool = False):
        L = lib()
        opts = pso_opts()
        opts.vmax = float(vmax)
        opts.device = int(device) if device >= 0 else 0  # < 0: the current device
        if stream is not None:
            opts.stream = int(getattr(stream, "cuda_stream", stream))
        opts.nccl_comm = nccl_comm
        opts.flags = ((PSO_FLAG_TIMING if timing else 0) | (PSO_FLAG_DEFER_INIT if defer_init else 0)
                      | (PSO_FLAG_ASYNC_GBEST if async_gbest else 0)
                      | (PSO_FLAG_COLUMN_SPLIT if column_split else 0)
                      | (PSO_FLAG_DEVICE if device >= 0 else 0)
                      | (PSO_FLAG_ALLREDUCE if allreduce_exchange else 0))
        opts.world, opts.rank = int(world), int(rank)
        if bounds is not None:  # per-dimension [vlo | vhi | xlo | xhi], 4 x d
            bounds = np.ascontiguousarray(bounds, dtype=np.float32).reshape(4 * int(d))
            opts.bounds = bounds.ctypes.data
        self._h = C.c_void_p()
        check(L.pso_create_ex(C.byref(self._h), int(n), int(d), float(w), float(c1), float(c2),
                              float(lo), float(hi), int(objective), int(seed) & (2**64 - 1),
                              C.byref(opts)), "pso_create_ex")
        info = self.info()
        self.n, self.d = int(n), int(d)
        self.n_local, self.row_begin = info["n_local"], info["row_begin"]
        self.rank, self.world = info["rank"], info["world"]
        # column split (NEXT-3): state and gbest position cover dims [col_begin, col_begin + d_local)
        self.column_split = bool(info["column_split"])
        self.col_begin, self.d_local = info["col_begin"], info["d_local"]
        self.vmax = float(np.float32(info["vmax"]))

    # -------------------------------------------------------------- lifecycle
    def close(self) -> None:
        if getattr(self, "_h", None) and self._h.value:
            lib().pso_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    @property
    def handle(self) -> C.c_void_p:
        return self._h

    # -------------------------------------------------------------- the path
    def init(self) -> "Swarm":
        """Deferred initialisation (defer_init=True): Alg. 1 lines 1-3."""
        check(lib().pso_init(self._h), "pso_init")
        return self

    def step(self, iters: int = 1) -> "Swarm":
        check(lib().pso_step(self._h, int(iters)), "pso_step")
        return self

    def synchronize(self) -> None:
        check(lib().pso_synchronize(self._h), "pso_synchronize")

    def gbest(self, pos: bool = True, out=None):
        """(fitness, global index, position or None) — synchronises."""
        f, i = C.c_float(), C.c_int64()
        buf = None
        if pos:
            buf = out if out is not None else np.empty(self.d_local, np.float32)
        check(lib().pso_get_gbest(self._h, C.byref(f), C.byref(i),
                                  _ptr(buf, self.d_local, writable=True)),
              "pso_get_gbest")
        return float(np.float32(f.value)), int(i.value), buf

    def get_state(self, out=None):
        """Rank-local (X, V, PB, pf, t) as dense host arrays — synchronises."""
        if out is None:
            m, d = self.n_local, self.d_local
            out = (np.empty((m, d), np.float32), np.empty((m, d), np.float32),
                   np.empty((m, d), np.float32), np.empty(m, np.float32))
        X, V, PB, pf = out
        t = C.c_uint64()
        m = self.n_local * self.d_local
        check(lib().pso_get_state(self._h, _ptr(X, m, writable=True), _ptr(V, m, writable=True),
                                  _ptr(PB, m, writable=True), _ptr(pf, self.n_local, writable=True),
                                  C.byref(t)),
              "pso_get_state")
        return X, V, PB, pf, int(t.value)

    def get_rows(self, rows):
        """(X, V, PB, pf) of the given rank-local rows (dense numpy arrays) without
        copying the rest of the swarm -- synchronises."""
        idx = np.ascontiguousarray(rows, dtype=np.int64).reshape(-1)
        m, d = idx.size, self.d_local
        X, V, PB = (np.empty((m, d), np.float32) for _ in range(3))
        pf = np.empty(m, np.float32)
        check(lib().pso_get_rows(self._h, idx.ctypes.data_as(C.POINTER(C.c_int64)), m,
                                 _ptr(X, m * d, writable=True), _ptr(V, m * d, writable=True),
                                 _ptr(PB, m * d, writable=True), _ptr(pf, m, writable=True)),
              "pso_get_rows")
        return X, V, PB, pf

    def set_state(self, X, V, PB, pf, t: int = 0) -> "Swarm":
        def prep(a):
            if hasattr(a, "data_ptr"):
                return a
            return np.ascontiguousarray(a, dtype=np.float32)
        X, V, PB, pf = prep(X), prep(V), prep(PB), prep(pf)
        dl = self.d_local
        for a, shape in ((X, (self.n_local, dl)), (V, (self.n_local, dl)),
                         (PB, (self.n_local, dl)), (pf, (self.n_local,))):
            if tuple(a.shape) != shape:
                raise ValueError(f"state shape {tuple(a.shape)} != {shape}")
        m = self.n_local * dl
        check(lib().pso_set_state(self._h, _ptr(X, m), _ptr(V, m), _ptr(PB, m),
                                  _ptr(pf, self.n_local), int(t)),
              "pso_set_state")
        return self

    def set_bounds(self, bounds) -> "Swarm":
        b = np.ascontiguousarray(bounds, dtype=np.float32).reshape(4 * self.d)
        check(lib().pso_set_bounds(self._h, C.c_void_p(b.ctypes.data)), "pso_set_bounds")
        return self

    def p2p_handle(self) -> tuple[bytes, int]:
        """(64-byte CUDA IPC handle of the arena, offset of the receive buffer)."""
        buf = C.create_string_buffer(64)
        off = C.c_uint64()
        check(lib().pso_p2p_handle(self._h, buf, C.byref(off)), "pso_p2p_handle")
        return buf.raw, int(off.value)

    def p2p_connect(self, handles, offsets) -> "Swarm":
        """Switch to the NVLink peer exchange (handles/offsets of every rank, in rank order)."""
        blob = C.create_string_buffer(b"".join(bytes(h) for h in handles), 64 * len(handles))
        offs = (C.c_uint64 * len(offsets))(*[int(o) for o in offsets])
        check(lib().pso_p2p_connect(self._h, blob, offs), "pso_p2p_connect")
        return self

    def p2p_probe(self, phase: int) -> bool:
        """Collective two-phase check of the mapped NVLink path (phase 0: store
        this rank's token into every peer; barrier; phase 1: True if every
        peer's token arrived)."""
        ok = C.c_int32(0)
        check(lib().pso_p2p_probe(self._h, int(phase), C.byref(ok)), "pso_p2p_probe")
        return bool(ok.value)

    def p2p_enable(self, on: bool = True) -> "Swarm":
        check(lib().pso_p2p_enable(self._h, int(bool(on))), "pso_p2p_enable")
        return self

    def info(self) -> dict:
        inf = pso_info()
        check(lib().pso_get_info(self._h, C.byref(inf)), "pso_get_info")
        return inf.as_dict()

    def reset_counters(self) -> None:
        check(lib().pso_reset_counters(self._h), "pso_reset_counters")


# ------------------------------------------------------------------ debug
def debug_philox(seed: int, tag: int, t: int, i: int, j0: int, m: int, use_curand=False,
                 device: int = -1) -> np.ndarray:
    out = np.empty(m, np.uint32)
    check(lib().pso_debug_philox(int(seed) & (2**64 - 1), tag, t, i, j0, m,
                                 out.ctypes.data_as(C.POINTER(C.c_uint32)), int(bool(use_curand)),
                                 int(device)), "pso_debug_philox")
    return out


def debug_objective(obj: int, X, device: int = -1) -> np.ndarray:
    X = np.ascontiguousarray(X, dtype=np.float32)
    if X.ndim == 1:
        X = X[None, :]
    out = np.empty(X.shape[0], np.float32)
    fp = C.POINTER(C.c_float)
    check(lib().pso_debug_objective(int(obj), X.ctypes.data_as(fp), X.shape[0], X.shape[1],
                                    out.ctypes.data_as(fp), int(device)), "pso_debug_objective")
    return out


# ------------------------------------------------------------------ NCCL plumbing
def nccl_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    check(lib().pso_nccl_get_unique_id(buf), "pso_nccl_get_unique_id")
    return buf.raw


def nccl_comm_init(world: int, uid: bytes, rank: int, device: int) -> int:
    comm = C.c_void_p()
    buf = C.create_string_buffer(bytes(uid), 128)
    check(lib().pso_nccl_comm_init(C.byref(comm), int(world), buf, int(rank), int(device)),
          "pso_nccl_comm_init")
    return comm.value


def nccl_comm_destroy(comm: int) -> None:
    check(lib().pso_nccl_comm_destroy(C.c_void_p(comm)), "pso_nccl_comm_destroy")
