exec > gpurun_out/check6.log 2>&1
WORKLOADS="W64K W256K" STEPS=200 bash tools/bench_sweep.sh
echo "== PSO_COL_STAGES=5"; PSO_COL_STAGES=5 WORKLOADS="W64K" STEPS=200 bash tools/bench_sweep.sh
timeout 1800 python -m pytest tests -m gpu -q -k "column or colsplit or col_ or decisions" 2>&1 | tail -15
compute-sanitizer --tool racecheck python -c "
import sys; sys.path.insert(0,'.')
import paper_conf_icpp_liuwc21_b200 as fp
for d, kw in ((20001, {}), (999, {'column_split': True})):
    s = fp.Swarm(5, d, 0.9, 2.0, 2.0, -5.12, 5.12, 3, 7, device=0, **kw); s.step(3); print(s.gbest()[:2]); s.close()
" 2>&1 | tail -3
