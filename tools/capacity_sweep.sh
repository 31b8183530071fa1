# C5 HBM-capacity sweep: Ackley d = 4096 with n = 1M, 2M, 2.9M on one B200
# (49, 98, 142.5 GB of state); kernel numbers only (no host checkpoint copy / CPU baseline).
for w in C5 C5_2M C5_2900K; do
  timeout 900 python bench.py --workload $w --steps ${STEPS:-30} --warmup 3 --no-e2e --no-cpu-baseline 2>&1 | tail -1 > gpurun_out/capacity_$w.json
  python - "$w" <<'PY'
import json, sys
w = sys.argv[1]
try:
    j = json.load(open(f"gpurun_out/capacity_{w}.json"))
except Exception:
    print(w, "FAILED", open(f"gpurun_out/capacity_{w}.json").read()[-400:]); sys.exit()
r = j["roofline"]
print(f"{w:9s} n={j['config']['n']:>8d} state {3*j['config']['n']*j['config']['d']*4/1e9:6.1f} GB  "
      f"{j['value']:.3e} upd/s  {j['ms_per_step']:8.3f} ms/step  {r['achieved']:6.0f} GB/s  frac {r['frac']:.3f}  clk {j['clocks']}")
PY
done
