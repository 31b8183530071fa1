for cfg in "" "PSO_VPT=1" "PSO_VPT=4" "PSO_STAGES=6" "PSO_STAGES=3" "PSO_CTAS=3" "PSO_CTAS=5" "PSO_VPT=4 PSO_CTAS=8" "PSO_PDL=0"; do
  echo "== $cfg"; env $cfg WORKLOADS="C3" STEPS=1000 bash tools/quick_perf.sh
done
