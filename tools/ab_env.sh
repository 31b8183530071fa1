# A/B a kernel knob: for each value of $VAR in $VALS, run tools/quick_perf.sh on $WORKLOADS.
# Example: VAR=PSO_L2PF VALS="0 2 4" WORKLOADS="C4 NS" bash tools/ab_env.sh
for v in ${VALS:-0}; do
  echo "== $VAR=$v"
  env $VAR=$v bash tools/quick_perf.sh
done
