"""ctypes binding of include/fastpso.h — argument marshalling only.

Every step of the hot path runs in the CUDA library ``libfastpso.so`` next to
this file.  There is no CPU fallback: importing the binding without the built
library raises.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libfastpso.so")

PSO_OK, PSO_ERR_INVALID, PSO_ERR_NOMEM, PSO_ERR_CUDA = 0, 1, 2, 3
PSO_ERR_NCCL, PSO_ERR_UNSUPPORTED, PSO_ERR_POISONED = 4, 5, 6
PSO_OBJ_SPHERE, PSO_OBJ_RASTRIGIN, PSO_OBJ_ROSENBROCK = 1, 2, 3
PSO_OBJ_GRIEWANK, PSO_OBJ_ACKLEY, PSO_OBJ_EASOM, PSO_OBJ_CUSTOM_BASE = 4, 5, 6, 64
PSO_FLAG_TIMING, PSO_FLAG_DEFER_INIT, PSO_FLAG_ASYNC_GBEST, PSO_FLAG_COLUMN_SPLIT = 1, 2, 4, 8
PSO_FLAG_DEVICE = 16
PSO_FLAG_ALLREDUCE = 32
PSO_D_MAX_ROW = 65536
PSO_D_AUTO_COLSPLIT = 9216
PSO_D_MAX = 1 << 24

# every symbol include/fastpso.h declares
EXPORTS = (
    "pso_create", "pso_create_ex", "pso_init", "pso_step", "pso_synchronize", "pso_get_gbest",
    "pso_get_state", "pso_get_rows", "pso_set_state", "pso_set_bounds", "pso_get_info", "pso_reset_counters", "pso_destroy",
    "pso_status_string", "pso_last_error", "pso_objective_registered",
    "pso_nccl_get_unique_id", "pso_nccl_comm_init", "pso_nccl_comm_destroy",
    "pso_p2p_handle", "pso_p2p_connect", "pso_p2p_probe", "pso_p2p_enable",
    "pso_debug_philox", "pso_debug_objective",
)


class pso_opts(C.Structure):
    _fields_ = [("vmax", C.c_float), ("device", C.c_int32), ("stream", C.c_void_p),
                ("nccl_comm", C.c_void_p), ("flags", C.c_uint32), ("world", C.c_int32),
                ("rank", C.c_int32), ("bounds", C.c_void_p)]


class pso_info(C.Structure):
    _fields_ = [
        ("n", C.c_int64), ("n_local", C.c_int64), ("row_begin", C.c_int64),
        ("d", C.c_int32), ("pitch", C.c_int32), ("rank", C.c_int32), ("world", C.c_int32),
        ("threads_per_cta", C.c_int32), ("vec_per_thread", C.c_int32), ("grid", C.c_int32),
        ("ctas_per_sm", C.c_int32), ("tma_pipeline", C.c_int32), ("pipeline_stages", C.c_int32),
        ("smem_bytes", C.c_int32), ("resident", C.c_int32), ("bounds", C.c_int32), ("cluster", C.c_int32),
        ("vmax", C.c_float), ("t", C.c_uint64),
        ("launches", C.c_uint64), ("improvements", C.c_uint64),
        ("pb_loads", C.c_uint64), ("pb_stores", C.c_uint64), ("lazy_pb", C.c_int32),
        ("step_kernel_ms", C.c_double), ("step_kernel_count", C.c_uint64),
        ("arena_bytes", C.c_size_t),
        ("column_split", C.c_int32), ("col_begin", C.c_int32), ("d_local", C.c_int32),
        ("col_tiles", C.c_int32),
    ]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class PsoError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        self.status = status
        super().__init__(f"{where}: {status_string(status)}: {detail}")


_lib = None


def lib() -> C.CDLL:
    """Load libfastpso.so (raises if it was not built: no fallback path exists)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"FastPSO CUDA library not built: {LIB_PATH} (run `make lib` or "
                          "`python -c 'import __graft_entry__ as g; g.build()'`)")
    L = C.CDLL(LIB_PATH, mode=C.RTLD_GLOBAL)
    H = C.c_void_p
    fp, i64p, u64p, u32p = (C.POINTER(C.c_float), C.POINTER(C.c_int64), C.POINTER(C.c_uint64),
                            C.POINTER(C.c_uint32))
    L.pso_create.argtypes = [C.POINTER(H), C.c_int64, C.c_int32, C.c_float, C.c_float, C.c_float,
                             C.c_float, C.c_float, C.c_int32, C.c_uint64]
    L.pso_create_ex.argtypes = L.pso_create.argtypes + [C.POINTER(pso_opts)]
    L.pso_step.argtypes = [H, C.c_int64]
    L.pso_init.argtypes = [H]
    L.pso_synchronize.argtypes = [H]
    L.pso_get_gbest.argtypes = [H, fp, i64p, C.c_void_p]
    L.pso_get_state.argtypes = [H, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, u64p]
    L.pso_get_rows.argtypes = [H, i64p, C.c_int64, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p]
    L.pso_set_state.argtypes = [H, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_uint64]
    L.pso_get_info.argtypes = [H, C.POINTER(pso_info)]
    L.pso_set_bounds.argtypes = [H, C.c_void_p]
    L.pso_reset_counters.argtypes = [H]
    L.pso_destroy.argtypes = [H]
    L.pso_destroy.restype = None
    L.pso_status_string.argtypes = [C.c_int]
    L.pso_status_string.restype = C.c_char_p
    L.pso_last_error.argtypes = []
    L.pso_last_error.restype = C.c_char_p
    L.pso_objective_registered.argtypes = [C.c_int32]
    L.pso_nccl_get_unique_id.argtypes = [C.c_void_p]
    L.pso_nccl_comm_init.argtypes = [C.POINTER(C.c_void_p), C.c_int32, C.c_void_p, C.c_int32,
                                     C.c_int32]
    L.pso_nccl_comm_destroy.argtypes = [C.c_void_p]
    L.pso_p2p_handle.argtypes = [H, C.c_void_p, u64p]
    L.pso_p2p_connect.argtypes = [H, C.c_void_p, u64p]
    L.pso_p2p_probe.argtypes = [H, C.c_int32, C.POINTER(C.c_int32)]
    L.pso_p2p_enable.argtypes = [H, C.c_int32]
    L.pso_debug_philox.argtypes = [C.c_uint64, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32,
                                   C.c_int64, u32p, C.c_int32, C.c_int32]
    L.pso_debug_objective.argtypes = [C.c_int32, fp, C.c_int64, C.c_int32, fp, C.c_int32]
    for name in EXPORTS:
        if name not in ("pso_destroy", "pso_status_string", "pso_last_error"):
            getattr(L, name).restype = C.c_int
    _lib = L
    return L


def status_string(s: int) -> str:
    return lib().pso_status_string(int(s)).decode()


def last_error() -> str:
    return lib().pso_last_error().decode()


def check(status: int, where: str) -> None:
    if status != PSO_OK:
        raise PsoError(status, where, last_error())
