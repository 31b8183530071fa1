# Per-SASS-instruction execution counts (ncu SourceCounters) of the step kernels:
# python-side summary in profiles/r02_sass_instruction_profile.json.
#   bash tools/sass_profile.sh            (WORKLOADS="NS C4 C3 W16K" by default)
mkdir -p gpurun_out
for w in ${WORKLOADS:-NS C4 C3 W16K}; do
  timeout 900 ncu --section SourceCounters --section InstructionStats --clock-control none --import-source on \
    -k regex:"k_step" -s 8 -c 1 -o /tmp/src_$w -f python bench.py --workload $w --steps 10 --warmup 5 \
    --no-e2e --no-cpu-baseline > /dev/null 2>&1
  ncu -i /tmp/src_$w.ncu-rep --page source --csv --print-source sass > gpurun_out/src_$w.csv 2>&1
done
