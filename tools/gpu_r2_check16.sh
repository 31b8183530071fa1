exec > gpurun_out/check16.log 2>&1
WORKLOADS="PAPER" STEPS=2000 bash tools/bench_sweep.sh
PSO_RESIDENT=0 WORKLOADS="C1" STEPS=2000 bash tools/bench_sweep.sh
timeout 1800 python -m pytest tests -m gpu -q -k "reg or both_kernels or single_step or decisions or resident or init" 2>&1 | tail -4
python tools/paper_table1.py
