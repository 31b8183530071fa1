# Round 2: column split with PDL (A/B), ring variants, C5 capacity sweep, column-split tests.
exec > gpurun_out/check5.log 2>&1
echo "== colsplit default (PDL)"; WORKLOADS="W64K W256K" STEPS=200 bash tools/bench_sweep.sh
echo "== PSO_PDL=0"; PSO_PDL=0 WORKLOADS="W64K" STEPS=200 bash tools/bench_sweep.sh
echo "== PSO_COL_CTAS=1"; PSO_COL_CTAS=1 PSO_COL_STAGES=6 WORKLOADS="W64K" STEPS=200 bash tools/bench_sweep.sh
echo "== PSO_COL_STAGES=2"; PSO_COL_STAGES=2 WORKLOADS="W64K" STEPS=200 bash tools/bench_sweep.sh
echo "== capacity"; bash tools/capacity_sweep.sh
timeout 1800 python -m pytest tests -m gpu -q -k "column or colsplit or col_" 2>&1 | tail -15
