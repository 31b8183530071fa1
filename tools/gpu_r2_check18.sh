exec > gpurun_out/check18.log 2>&1
WORKLOADS="W64K W256K W64K" STEPS=200 bash tools/bench_sweep.sh
timeout 1800 python -m pytest tests -m gpu -q -k "column or colsplit or col_ or maximum" 2>&1 | tail -4
