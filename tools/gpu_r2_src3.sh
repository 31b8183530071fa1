exec > gpurun_out/src3.log 2>&1
timeout 900 ncu --section SourceCounters --section InstructionStats --section WarpStateStats --clock-control none --import-source on -k regex:"k_gridres" -c 1 -o /tmp/src_C2 -f python bench.py --workload C2 --steps 200 --warmup 5 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu -i /tmp/src_C2.ncu-rep --page source --csv --print-source sass > gpurun_out/src_C2.csv 2>&1
ncu -i /tmp/src_C2.ncu-rep --page details --csv > gpurun_out/det_C2.csv 2>&1
