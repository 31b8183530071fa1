exec > gpurun_out/check9.log 2>&1
python - <<'PY'
import os, paper_conf_icpp_liuwc21_b200 as fp
from synth import WORKLOADS
w = WORKLOADS["W16K"]
for env in ({"PSO_CLUSTER": "8", "PSO_VPT": "2", "PSO_CTAS": "2"}, {"PSO_CLUSTER": "4", "PSO_VPT": "4"}, {"PSO_CLUSTER": "8", "PSO_VPT": "2"}):
    os.environ.update(env)
    try:
        s = fp.Swarm(w.n, w.d, w.w, w.c1, w.c2, w.lo, w.hi, w.objective, w.seed, device=0)
        i = s.info(); print(env, "cluster", i["cluster"], "grid", i["grid"], "stages", i["pipeline_stages"], "vpt", i["vec_per_thread"], "threads", i["threads_per_cta"], "smem", i["smem_bytes"]); s.close()
    except Exception as e:
        print(env, "FAILED", e)
    for k in env: os.environ.pop(k)
PY
echo "== C8 VPT2 CTAS2"; PSO_CLUSTER=8 PSO_VPT=2 PSO_CTAS=2 WORKLOADS="W16K" STEPS=200 bash tools/bench_sweep.sh
echo "== C4 VPT4"; PSO_CLUSTER=4 PSO_VPT=4 WORKLOADS="W16K" STEPS=200 bash tools/bench_sweep.sh
echo "== C8 VPT2"; PSO_CLUSTER=8 PSO_VPT=2 WORKLOADS="W16K" STEPS=200 bash tools/bench_sweep.sh
echo "== default"; WORKLOADS="W16K" STEPS=200 bash tools/bench_sweep.sh
