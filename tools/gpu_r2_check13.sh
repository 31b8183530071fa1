exec > gpurun_out/check13.log 2>&1
WORKLOADS="C4 NS C2 C5" STEPS=300 bash tools/bench_sweep.sh
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -6
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
