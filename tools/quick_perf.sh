# Kernel-time check of a few workloads (no e2e / cpu baseline): one line each.
for w in ${WORKLOADS:-C3 C4 NS}; do
  timeout 300 python bench.py --workload $w --steps ${STEPS:-300} --warmup 10 --no-e2e --no-cpu-baseline 2>&1 | tail -1 | python -c "
import json,sys
j=json.loads(sys.stdin.read()); r=j['roofline']
print('$w', f\"{j['ms_per_step']*1e3:8.2f} us/step kern {r['kernel_avg_us']:8.2f} us {r['achieved']:6.0f} GB/s frac {r['frac']:.3f} cta {r['cta'].get('threads')}x{r['cta'].get('grid')} st {r['cta'].get('stages')} clk {j['clocks']['sm_mhz']} {j['clocks']['reasons']}\")" || echo "$w FAILED"
done
