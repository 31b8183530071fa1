exec > gpurun_out/check19.log 2>&1
WORKLOADS="W64K W256K" STEPS=200 bash tools/bench_sweep.sh
for w in W64K W256K; do cp gpurun_out/sweep_$w.json gpurun_out/r02_final_sweep_$w.json; done
timeout 1800 python -m pytest tests -m gpu -q -k "column or colsplit or col_ or maximum" 2>&1 | tail -3
timeout 900 ncu --set full --metrics lts__t_bytes.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:"k_col_step" -s 8 -c 1 -o /tmp/prof_W64K -f python bench.py --workload W64K --steps 10 --warmup 5 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python tools/ncu_summary.py /tmp/prof_W64K.ncu-rep > gpurun_out/ncu_summary_W64K_final.txt 2>&1
cat gpurun_out/ncu_summary_W64K_final.txt
