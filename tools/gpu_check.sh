# GPU-box check: smoke, GPU tests, a short bench, ncu launch list + one full capture.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 1200 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS:-} 2>&1 | tail -40
timeout 600 python bench.py --steps 1000 --warmup 20 2>&1 | tail -3 > gpurun_out/bench.json
cat gpurun_out/bench.json
if [ -n "$NCU" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv \
    --log-file gpurun_out/launches.csv python bench.py --steps 40 --warmup 5 --no-e2e --no-cpu-baseline > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_step -s 8 -c 1 \
    -o gpurun_out/prof_step python bench.py --steps 10 --warmup 5 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
  tail -3 gpurun_out/ncu_full.log
fi
