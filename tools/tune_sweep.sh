# Launch-shape sweep of the TMA step kernel on the north-star swarm (kernel time only).
W=${W:-NS}
for cfg in "2 2 0" "2 1 0" "4 2 0" "4 3 0" "4 4 0" "2 2 3" "2 2 2" "1 2 0"; do
  set -- $cfg
  PSO_VPT=$1 PSO_CTAS=$2 PSO_STAGES=$3 timeout 300 python bench.py --workload $W --steps 300 --warmup 10 --no-e2e --no-cpu-baseline 2>&1 | tail -1 | python -c "
import json,sys
j=json.loads(sys.stdin.read()); r=j['roofline']
print('vpt=$1 ctas=$2 stages=$3', f\"{r['kernel_avg_us']:8.1f} us {r['achieved']:6.0f} GB/s frac {r['frac']:.3f} cta {r['cta']} clk {j['clocks']['sm_mhz']} {j['clocks']['reasons']}\")" || echo "vpt=$1 ctas=$2 stages=$3 FAILED"
done
