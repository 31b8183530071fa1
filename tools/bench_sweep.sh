# Bench every workload on one GPU (kernel numbers; no e2e / cpu baseline).
for w in ${WORKLOADS:-C1 C2 C3 C4 NS C5}; do
  timeout 600 python bench.py --workload $w --steps ${STEPS:-500} --warmup 10 --no-e2e --no-cpu-baseline 2>&1 | tail -1 > gpurun_out/sweep_$w.json
  python - "$w" <<'PY'
import json, sys
w = sys.argv[1]
try:
    j = json.load(open(f"gpurun_out/sweep_{w}.json"))
except Exception as e:
    print(w, "FAILED", open(f"gpurun_out/sweep_{w}.json").read()[-300:]); sys.exit()
r = j["roofline"]
print(f"{w:4s} {j['config']['workload']:34s} {j['value']:.3e} upd/s  {j['ms_per_step']*1e3:9.1f} us/step  "
      f"kern {r['kernel_avg_us']:9.1f} us  {r['achieved']:7.0f} GB/s  frac {r['frac']:.3f}  "
      f"cta {r['cta']}  clk {j['clocks']}")
PY
done
