"""The C-ABI boundary on a GPU-less host: the library loads, exports every
symbol include/fastpso.h declares, and validates arguments (returning status
codes, never aborting) before it touches a device."""
import ctypes as C
import os
import re

import pytest

import paper_conf_icpp_liuwc21_b200 as fp
from paper_conf_icpp_liuwc21_b200 import _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    src = open(os.path.join(ROOT, "include", "fastpso.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(pso_[a-z_0-9]+)\s*\(", src)))


def test_header_and_binding_agree():
    syms = header_symbols()
    assert len(syms) >= 18
    assert sorted(_lib.EXPORTS) == syms


def test_header_limits_match_binding():
    src = open(os.path.join(ROOT, "include", "fastpso.h")).read()
    for name in ("PSO_D_MAX_ROW", "PSO_D_AUTO_COLSPLIT"):
        m = re.search(r"#define\s+%s\s+(\d+)" % name, src)
        assert m and int(m.group(1)) == getattr(_lib, name), name
    assert re.search(r"#define\s+PSO_D_MAX\s+\(1 << 24\)", src) and _lib.PSO_D_MAX == 1 << 24


def test_library_exports_every_declared_symbol():
    L = fp.lib()
    for s in header_symbols():
        assert hasattr(L, s), s


def test_library_is_sm100a_only():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", _lib.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out
    assert all("sm_100a" in line for line in out.splitlines() if line.strip())


def test_fused_kernel_uses_bulk_async_copy():
    import subprocess
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", _lib.LIB_PATH],
                          capture_output=True, text=True).stdout
    assert "UBLKCP" in sass  # cp.async.bulk staging of gbest into shared memory
    assert "LDG.E.128" in sass and "STG.E.128" in sass  # 128-bit streaming


def _create(n=10, d=10, w=0.9, c1=2.0, c2=2.0, lo=-1.0, hi=1.0, obj=1, seed=1, opts=None):
    h = C.c_void_p(123)
    L = fp.lib()
    if opts is None:
        st = L.pso_create(C.byref(h), n, d, w, c1, c2, lo, hi, obj, seed)
    else:
        st = L.pso_create_ex(C.byref(h), n, d, w, c1, c2, lo, hi, obj, seed, C.byref(opts))
    return st, h


@pytest.mark.parametrize("kw,status", [
    (dict(n=0), 1), (dict(n=2**32), 1), (dict(d=0), 1), (dict(d=2**24 + 1), 5),
    (dict(lo=1.0, hi=1.0), 1), (dict(lo=2.0, hi=1.0), 1), (dict(hi=float("inf")), 1),
    (dict(w=float("nan")), 1), (dict(c1=float("inf")), 1), (dict(obj=0), 1), (dict(obj=63), 1),
])
def test_invalid_arguments_return_status(kw, status):
    st, h = _create(**kw)
    assert st == status, fp.last_error()
    assert h.value is None  # *out is cleared on failure
    assert fp.last_error()


def test_column_split_validation_before_any_device_call():
    o = _lib.pso_opts()
    o.device = -1
    o.flags = fp.PSO_FLAG_COLUMN_SPLIT | _lib.PSO_FLAG_ASYNC_GBEST
    assert _create(opts=o)[0] == 1 and "ASYNC" in fp.last_error()
    # rows beyond the row kernels with a particle split: needs the column split
    o = _lib.pso_opts()
    o.device = -1
    o.world, o.rank, o.flags = 2, 0, _lib.PSO_FLAG_DEFER_INIT
    assert _create(d=65537, opts=o)[0] == 5 and "COLUMN_SPLIT" in fp.last_error()


def test_invalid_flags_and_vmax():
    o = _lib.pso_opts()
    o.flags = 0x80
    o.device = -1
    assert _create(opts=o)[0] == 1
    o = _lib.pso_opts()
    o.vmax = float("nan")
    assert _create(opts=o)[0] == 1


def test_null_handle_calls():
    L = fp.lib()
    assert L.pso_step(None, 1) == 1
    assert L.pso_synchronize(None) == 1
    assert L.pso_get_gbest(None, None, None, None) == 1
    assert L.pso_get_state(None, None, None, None, None, None) == 1
    assert L.pso_set_state(None, None, None, None, None, 0) == 1
    assert L.pso_get_info(None, None) == 1
    L.pso_destroy(None)  # NULL-safe
    assert L.pso_create(None, 1, 1, 0, 0, 0, 0, 1, 1, 0) == 1


def test_status_strings():
    for s, name in enumerate(["PSO_OK", "PSO_ERR_INVALID", "PSO_ERR_NOMEM", "PSO_ERR_CUDA",
                              "PSO_ERR_NCCL", "PSO_ERR_UNSUPPORTED", "PSO_ERR_POISONED"]):
        assert fp.status_string(s) == name


def test_objective_registry():
    for obj in (1, 2, 3, 4, 5, 6):
        assert fp.objective_registered(obj)
    for obj in (0, 7, 63, 64, -1):
        assert not fp.objective_registered(obj)


def test_valid_create_without_gpu_reports_cuda_error():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    st, h = _create()
    assert st == 3 and h.value is None
    assert "cuda" in fp.last_error().lower()


def test_product_path_fails_loudly_without_library(monkeypatch, tmp_path):
    monkeypatch.setattr(_lib, "LIB_PATH", str(tmp_path / "missing.so"))
    monkeypatch.setattr(_lib, "_lib", None)
    with pytest.raises(ImportError):
        _lib.lib()


def test_bounds_validation_without_gpu():
    import numpy as np
    o = _lib.pso_opts()
    o.device = -1
    b = np.zeros(4 * 10, np.float32)
    b[10:20] = 1.0   # vhi
    b[20:30] = -1.0  # xlo
    b[30:40] = 1.0   # xhi
    b[25] = 2.0      # xlo > xhi at dim 5
    o.bounds = b.ctypes.data
    assert _create(opts=o)[0] == 1
    b[25] = -1.0
    b[3] = np.nan
    assert _create(opts=o)[0] == 1


def test_device_flag_validation_without_gpu():
    """pso_opts.device is read only with PSO_FLAG_DEVICE (zero-initialised opts
    are the defaults: the caller's current device); a negative ordinal with
    the flag is rejected before any device call."""
    o = _lib.pso_opts()
    o.flags = _lib.PSO_FLAG_DEVICE
    o.device = -2
    assert _create(opts=o)[0] == 1 and "PSO_FLAG_DEVICE" in fp.last_error()


def test_host_buffer_validation():
    """The binding checks element type and count of every host buffer the
    library reads or writes (no silent reinterpretation, no overflow)."""
    import numpy as np
    import torch
    from paper_conf_icpp_liuwc21_b200 import _ptr
    assert _ptr(None) is None
    assert _ptr(np.zeros(6, np.float32), 6).value
    assert _ptr(torch.zeros(2, 3), 6).value
    for bad, count in ((np.zeros(6, np.float64), 6), (np.zeros(5, np.float32), 6),
                       (torch.zeros(6, dtype=torch.float16), 6), (torch.zeros(7), 6),
                       (torch.zeros(6, dtype=torch.float64), None), (np.zeros((6, 2), np.float32)[:, 0], 6)):
        with pytest.raises(ValueError):
            _ptr(bad, count)
    ro = np.zeros(3, np.float32)
    ro.flags.writeable = False
    with pytest.raises(ValueError):
        _ptr(ro, 3, writable=True)


def test_header_flags_and_objectives_match_binding():
    src = open(os.path.join(ROOT, "include", "fastpso.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    consts = dict((k, int(v)) for k, v in re.findall(r"\b(PSO_(?:FLAG|OBJ)_[A-Z_]+)\s*=\s*(\d+)", src))
    assert len(consts) >= 13
    for k, v in consts.items():
        assert getattr(_lib, k) == v, k
    flags = [v for k, v in consts.items() if k.startswith("PSO_FLAG_")]
    assert all(f & (f - 1) == 0 for f in flags) and len(set(flags)) == len(flags)
