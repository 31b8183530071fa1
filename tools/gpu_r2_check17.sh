exec > gpurun_out/check17.log 2>&1
echo "== warp (default)"; WORKLOADS="PAPER" STEPS=2000 bash tools/bench_sweep.sh
echo "== reg"; PSO_KERNEL=reg PSO_RESIDENT=0 WORKLOADS="PAPER" STEPS=2000 bash tools/bench_sweep.sh
timeout 1800 python -m pytest tests -m gpu -q -x -k "warp_per_row or resident or single_step or decisions or init or exchange or lockstep or end_to_end" 2>&1 | tail -5
python tools/paper_table1.py
