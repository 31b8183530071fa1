exec > gpurun_out/check15.log 2>&1
echo "== default"; WORKLOADS="PAPER" STEPS=2000 bash tools/bench_sweep.sh
echo "== tma"; PSO_KERNEL=tma WORKLOADS="PAPER" STEPS=2000 bash tools/bench_sweep.sh
W=PAPER STEPS=2000 CFGS="1,0,0 2,0,0 1,1,0 1,2,0 1,4,0 1,8,0" bash tools/tune_sweep.sh
