for cfg in "0 0" "8 2" "4 2" "8 1" "16 1" "2 1"; do
  set -- $cfg
  PSO_CLUSTER=$1 PSO_CTAS=$2 WORKLOADS="${W:-W16K}" bash tools/quick_perf.sh | sed "s/^/cl=$1 ctas=$2 /"
done
