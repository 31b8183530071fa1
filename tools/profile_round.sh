# Round profile refresh on one GPU: default bench line (e2e + cpu baseline),
# the reference (oracle) arm, a kernel sweep of every workload, the ncu launch
# list of the default bench and one ncu --set full capture per workload.
# Output: gpurun_out/prof/ (summarise here with tools/ncu_summary.py).
set -x
O=gpurun_out/prof
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/gpu.txt
python tools/hbm_mix_probe.py > $O/hbm_mix_probe.json 2>&1
timeout 900 python bench.py 2>&1 | tail -1 > $O/bench_default.json
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 2>&1 | tail -1 > $O/bench_reference.json
for w in ${WORKLOADS:-C1 C2 C3 C4 NS C5 W16K W64K}; do
  st=500; [ $w = C5 ] && st=100
  timeout 600 python bench.py --workload $w --steps $st --warmup 10 --no-e2e --no-cpu-baseline 2>&1 | tail -1 > $O/sweep_$w.json
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv \
  --log-file $O/launches_northstar.csv python bench.py --steps 30 --warmup 5 --no-e2e --no-cpu-baseline > /dev/null 2>&1
# the .ncu-rep files stay on the box (gpurun copies back <= 64 MiB); their summaries come back
R=${NCU_REP_DIR:-/tmp/ncu_reps}
mkdir -p $R
for w in ${NCU_WORKLOADS:-NS C4 C3 C5 W16K W64K}; do
  timeout 900 ncu --set full --metrics lts__t_bytes.sum,lts__t_sector_hit_rate.pct --clock-control none --import-source on -k regex:"k_step|k_col_step" -s 8 -c 1 \
    -o $R/prof_$w -f python bench.py --workload $w --steps 10 --warmup 5 --no-e2e --no-cpu-baseline > $O/ncu_$w.log 2>&1
  python tools/ncu_summary.py $R/prof_$w.ncu-rep > $O/ncu_summary_$w.txt 2>&1
done
ls -la $O
