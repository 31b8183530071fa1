# Round 2: pipelined cluster finaliser -- W16K sweep and the cluster parity tests.
exec > gpurun_out/check4.log 2>&1
set -x
WORKLOADS="W16K" STEPS=200 bash tools/bench_sweep.sh
for C in 2 8; do echo "== PSO_CLUSTER=$C"; PSO_CLUSTER=$C WORKLOADS="W16K" STEPS=200 bash tools/bench_sweep.sh; done
timeout 1800 python -m pytest tests -m gpu -q -k "cluster or wide or W16K or decisions or multirank or 10000 or sharing" 2>&1 | tail -30
