# Bench lines of the heavier workloads at the start of a call (no test suite before them, so the
# board is not yet at its power cap): gpurun_out/fresh/sweep_<W>.json.
mkdir -p gpurun_out/fresh
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/fresh/gpu.txt
for w in ${WORKLOADS:-W16K W64K W256K C4 NS C3 C5}; do
  st=500; [ $w = C5 ] && st=100
  timeout 600 python bench.py --workload $w --steps $st --warmup 10 --no-e2e --no-cpu-baseline 2>&1 | tail -1 > gpurun_out/fresh/sweep_$w.json
  sleep 5
done
