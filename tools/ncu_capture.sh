# One ncu --set full capture of the step kernel per workload (single GPU), plus a launch list.
for W in ${WORKLOADS:-NS}; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_step -s 8 -c 1 \
    -o gpurun_out/prof_$W python bench.py --workload $W --steps 10 --warmup 5 --no-e2e --no-cpu-baseline > gpurun_out/ncu_$W.log 2>&1
  tail -1 gpurun_out/ncu_$W.log | cut -c1-100
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 30 --warmup 5 --no-e2e --no-cpu-baseline > /dev/null 2>&1
