exec > gpurun_out/exp3.log 2>&1
for h in 0 1 0 1; do echo "== PSO_L2HINT=$h"; PSO_L2HINT=$h WORKLOADS="C3 C2x" STEPS=1000 bash tools/bench_sweep.sh 2>/dev/null | grep -v FAILED; done
for h in 0 1; do echo "== PSO_L2HINT=$h"; PSO_L2HINT=$h WORKLOADS="NS C4" STEPS=300 bash tools/bench_sweep.sh; done
