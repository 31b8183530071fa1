# Round 2: cluster-size A/B on W16K, then the full GPU suite.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python - <<'PY'
import paper_conf_icpp_liuwc21_b200 as fp
from synth import WORKLOADS
for name in ("W16K",):
    w = WORKLOADS[name]
    s = fp.Swarm(w.n, w.d, w.w, w.c1, w.c2, w.lo, w.hi, w.objective, w.seed, device=0)
    i = s.info(); print(name, "cluster", i["cluster"], "grid", i["grid"], "stages", i["pipeline_stages"], "vpt", i["vec_per_thread"], "threads", i["threads_per_cta"]); s.close()
PY
WORKLOADS="W16K" STEPS=200 bash tools/bench_sweep.sh
PSO_CLUSTER_POW2=1 WORKLOADS="W16K" STEPS=200 bash tools/bench_sweep.sh
for C in 3 5 6; do PSO_CLUSTER=$C WORKLOADS="W16K" STEPS=200 bash tools/bench_sweep.sh; done
timeout 2400 python -m pytest tests -m gpu -q -x 2>&1 | tail -30 > gpurun_out/full.log
tail -30 gpurun_out/full.log
