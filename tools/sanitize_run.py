"""Small runs of every kernel path, for compute-sanitizer (memcheck / racecheck / synccheck).

Paths: register streaming and TMA pipeline (eager and lazy pbest rows, L2 prefetch, serpentine
order), the CTA-resident and grid-resident latency kernels, the thread-block cluster, the column
split (forced and automatic), per-dimension bounds, and the gbest exchange on a 1-rank NCCL
communicator (records, merge in the next prologue, select kernel).
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import paper_conf_icpp_liuwc21_b200 as fp  # noqa: E402
from synth import DOMAINS  # noqa: E402


def run(tag, obj, n, d, steps=3, env=None, **kw):
    saved = {k: os.environ.get(k) for k in (env or {})}
    os.environ.update(env or {})
    try:
        lo, hi = DOMAINS[obj]
        s = fp.Swarm(n, d, 0.9, 2.0, 2.0, lo, hi, obj, 7, device=0, **kw)
        s.step(steps)
        f, i, _ = s.gbest()
        X, V, PB, pf, t = s.get_state()
        info = s.info()
        path = ("colsplit" if info["column_split"] else "cluster" if info["cluster"] else
                ["", "cta-resident", "grid-resident", "persistent"][info["resident"]] if info["resident"] else
                "tma" if info["tma_pipeline"] else "reg")
        print(f"{tag:14s} obj={obj} n={n} d={d} path={path} lazy={info['lazy_pb']} f={f:.6g} i={i} "
              f"t={t}", flush=True)
        s.close()
    finally:
        for k, v in saved.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


for kernel in ("reg", "tma"):
    for obj, n, d in ((2, 40, 1000), (3, 33, 999), (4, 20, 2000), (5, 7, 4096), (1, 5, 13)):
        run(kernel, obj, n, d, env={"PSO_KERNEL": kernel, "PSO_RESIDENT": "0"})
run("lazy+prefetch", 4, 300, 2000, steps=4, env={"PSO_RESIDENT": "0", "PSO_L2PF_ALL": "1"})
run("cta-resident", 1, 32, 10, steps=10)
run("grid-resident", 2, 256, 1000, steps=5)
run("persistent", 3, 3000, 1000, steps=5, env={"PSO_PERSIST": "1"})
run("persistent-few", 1, 60, 2001, steps=4, env={"PSO_PERSIST": "1"})
run("cluster", 3, 5, 12000, steps=3, env={"PSO_CLUSTER": "4"})
run("cluster-C16", 4, 3, 40000, steps=2, env={"PSO_CLUSTER": "16"})
run("colsplit-auto", 2, 3, 20001, steps=3)
run("colsplit", 3, 9, 999, steps=3, column_split=True)
run("colsplit-auto2", 4, 6, 12000, steps=3)
# position/pbest slots through every transition (mixed improvements), G cache over 9 tiles
run("colsplit-slots", 1, 40, 2049, steps=8, column_split=True, vmax=2.0)
bw = np.stack([np.full(12000, -0.5, np.float32), np.full(12000, 0.5, np.float32),
               np.full(12000, -2.0, np.float32), np.full(12000, 2.0, np.float32)])
run("colsplit-bounds", 3, 6, 12000, steps=3, bounds=bw)
b = np.stack([np.full(1000, -0.5, np.float32), np.full(1000, 0.5, np.float32),
              np.full(1000, -3.0, np.float32), np.full(1000, 4.0, np.float32)])
run("bounds", 2, 40, 1000, steps=3, bounds=b)
comm = fp.nccl_comm_init(1, fp.nccl_unique_id(), 0, 0)
try:
    run("exchange-nccl", 2, 300, 1000, steps=3, env={"PSO_FORCE_EXCHANGE": "1"}, nccl_comm=comm)
    # runs of 4 iterations replay the captured [step, all-gather] CUDA graph
    run("nccl-graph", 2, 300, 1000, steps=11, env={"PSO_FORCE_EXCHANGE": "1"}, nccl_comm=comm)
    # NVLink records on a 1-rank group: IPC mapping, connect probe, peer stores
    os.environ["PSO_FORCE_EXCHANGE"] = "1"
    lo, hi = DOMAINS[2]
    s = fp.Swarm(300, 1000, 0.9, 2.0, 2.0, lo, hi, 2, 7, device=0, nccl_comm=comm)
    h, off = s.p2p_handle()
    s.p2p_connect([h], [off])
    s.p2p_probe(0)
    assert s.p2p_probe(1)
    s.p2p_enable(True)
    s.step(3)
    print("p2p-probe      f=%.6g i=%d" % s.gbest()[:2], flush=True)
    s.close()
    os.environ.pop("PSO_FORCE_EXCHANGE")
finally:
    fp.nccl_comm_destroy(comm)
print("sanitize_run done", flush=True)
