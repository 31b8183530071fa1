# C2 (grid-resident) launch-shape sweep.
exec > gpurun_out/check12.log 2>&1
W=C2 STEPS=2000 CFGS="0,0,0 0,1,0 0,2,0 0,3,0 1,1,0 1,2,0 4,1,0" bash tools/tune_sweep.sh
