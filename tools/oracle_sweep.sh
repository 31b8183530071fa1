# The oracle (the reference arm) beside every configuration, on the GPU box's host:
# C1 and C2 in full (whole pso_step(T) runs), the others as bounded samples of the same workload.
for w in C1 C2 C3 C4 NS C5; do
  timeout 600 python bench.py --impl reference --workload $w --steps 3 --warmup 1 --ref-seconds 20 2>&1 | tail -1 > gpurun_out/oracle_$w.json
done
python - <<'PY'
import os, sys, time, json
sys.path.insert(0, ".")
import oracle as orc
from synth import WORKLOADS
for key in ("C1", "C2"):
    w = WORKLOADS[key]
    s = orc.OracleSwarm(w.n, w.d, w.w, w.c1, w.c2, w.lo, w.hi, w.objective, w.seed, vmax=w.vmax)
    t0 = time.perf_counter(); s.step(w.iters); dt = time.perf_counter() - t0
    print(json.dumps({"workload": w.name, "full_run_iterations": w.iters, "seconds": dt,
                      "updates_per_s": w.n * w.d * w.iters / dt, "gbest": s.gf, "cores": 1}))
PY
