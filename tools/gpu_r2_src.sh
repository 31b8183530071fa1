# Source-level (SASS) instruction counts of the C4 and W16K step kernels.
exec > gpurun_out/src.log 2>&1
for w in C4 W16K; do
  timeout 900 ncu --section SourceCounters --section InstructionStats --clock-control none --import-source on -k regex:"k_step" -s 8 -c 1 -o /tmp/src_$w -f python bench.py --workload $w --steps 10 --warmup 5 --no-e2e --no-cpu-baseline > /dev/null 2>&1
  ncu -i /tmp/src_$w.ncu-rep --page source --csv --print-source sass > gpurun_out/src_$w.csv 2>&1
  ls -la gpurun_out/src_$w.csv
done
