exec > gpurun_out/check14.log 2>&1
python - <<'PY'
import os, paper_conf_icpp_liuwc21_b200 as fp
from synth import WORKLOADS
w = WORKLOADS["PAPER"]
for v in ("1", "0"):
    os.environ["PSO_GRIDRES_SMALL"] = v
    s = fp.Swarm(w.n, w.d, w.w, w.c1, w.c2, w.lo, w.hi, w.objective, w.seed, device=0)
    i = s.info(); print(v, "resident", i["resident"], "grid", i["grid"], "threads", i["threads_per_cta"], "smem", i["smem_bytes"]); s.close()
PY
for v in 1 0; do echo "== PSO_GRIDRES_SMALL=$v"; PSO_GRIDRES_SMALL=$v WORKLOADS="PAPER" STEPS=2000 bash tools/bench_sweep.sh; done
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "grid_resident or decisions" 2>&1 | tail -5
timeout 1200 python -m pytest tests/test_gpu_edge_cases.py -m gpu -q 2>&1 | tail -3
python tools/paper_table1.py
