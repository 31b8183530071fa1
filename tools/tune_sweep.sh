# Launch-shape sweep of the TMA step kernel (kernel time only).
# W = workload, CFGS = "vpt,ctas,stages ..." (0 = automatic).
W=${W:-NS}
for cfg in ${CFGS:-2,2,0 2,1,0 4,2,0 4,3,0 4,4,0 2,2,3 1,2,0}; do
  IFS=, read v c st <<< "$cfg"
  PSO_VPT=$v PSO_CTAS=$c PSO_STAGES=$st timeout 300 python bench.py --workload $W --steps ${STEPS:-300} --warmup 10 --no-e2e --no-cpu-baseline 2>&1 | tail -1 | python -c "
import json,sys
j=json.loads(sys.stdin.read()); r=j['roofline']
print('$W vpt=$v ctas=$c stages=$st', f\"{r['kernel_avg_us']:8.1f} us {r['achieved']:6.0f} GB/s frac {r['frac']:.3f} cta {r['cta']} clk {j['clocks']['sm_mhz']} {j['clocks']['reasons']}\")" || echo "$W vpt=$v ctas=$c stages=$st FAILED"
done
