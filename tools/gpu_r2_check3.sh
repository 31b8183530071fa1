# Round 2: W16K cluster sizes, reading sweeps, default bench, then the full GPU suite.
exec > gpurun_out/check3.log 2>&1
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python - <<'PY'
import paper_conf_icpp_liuwc21_b200 as fp
from synth import WORKLOADS
w = WORKLOADS["W16K"]
s = fp.Swarm(w.n, w.d, w.w, w.c1, w.c2, w.lo, w.hi, w.objective, w.seed, device=0)
i = s.info(); print("W16K auto: cluster", i["cluster"], "grid", i["grid"], "stages", i["pipeline_stages"], "vpt", i["vec_per_thread"], "threads", i["threads_per_cta"]); s.close()
PY
WORKLOADS="W16K" STEPS=200 bash tools/bench_sweep.sh
for C in 3 4 5 8; do echo "== PSO_CLUSTER=$C"; PSO_CLUSTER=$C WORKLOADS="W16K" STEPS=200 bash tools/bench_sweep.sh; done
WORKLOADS="C4_V600 NS_V512 C4 NS" STEPS=500 bash tools/bench_sweep.sh
for w in C4_V600 NS_V512; do cp gpurun_out/sweep_$w.json gpurun_out/r02_sweep_$w.json; done
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -30
