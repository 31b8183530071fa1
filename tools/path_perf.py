"""Host-timed comparison of step paths on one GPU (experiments, not bench numbers):
python tools/path_perf.py W64K W16K  -> default path vs the column split, us/iteration."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_liuwc21_b200 as fp  # noqa: E402
from synth import WORKLOADS  # noqa: E402


def run(w, K, **kw):
    s = fp.Swarm(w.n, w.d, w.w, w.c1, w.c2, w.lo, w.hi, w.objective, w.seed, vmax=w.vmax,
                 device=0, **kw)
    s.step(5)
    s.synchronize()
    t0 = time.perf_counter()
    s.step(K)
    s.synchronize()
    dt = (time.perf_counter() - t0) / K
    info = s.info()
    s.close()
    return dt, info


for name in sys.argv[1:] or ["W64K", "W16K"]:
    if name in WORKLOADS:
        w = WORKLOADS[name]
    else:  # ad hoc: <workload>:<n>x<d>, e.g. W64K:8192x32768
        base, shape = name.split(":")
        n, d = (int(v) for v in shape.split("x"))
        w = WORKLOADS[base].with_(n=n, d=d)
    kws = [{}] if w.d > fp.PSO_D_MAX_ROW else [{}, {"column_split": True}]
    for kw in kws:
        dt, info = run(w, int(os.environ.get("K", "100")), **kw)
        bpu = 20.0
        print(f"{name:6s} {str(kw):24s} {dt * 1e6:9.1f} us/iter  {w.n * w.d / dt:.3e} upd/s  "
              f"~{bpu * w.n * w.d / dt / 1e9:6.0f} GB/s@20B  cluster={info.get('cluster')} "
              f"col_tiles={info.get('col_tiles')}", flush=True)
