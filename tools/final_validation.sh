# Round 2 final validation on one B200: smoke, the GPU suite, the driver's bench command,
# the N > 1 path as 8 ranks sharing GPU 0 (harness check, not a scaling number), then the
# profile refresh (bench lines, sweeps, ncu).  (compute-sanitizer is closed on this pool since
# the end of round 2: tools/gpu_sanitize.sh is kept for pools where it is allowed.)
mkdir -p gpurun_out/final
exec > gpurun_out/final/log.txt 2>&1
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -15
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 2>&1 | tail -1 > gpurun_out/final/bench_driver_cmd.json
PSO_SHARE_GPU=1 PSO_QUIET=1 timeout 900 python bench.py --gpus 8 --steps 50 --warmup 5 --workload NS 2>/dev/null | grep '^{' > gpurun_out/final/bench_8ranks_shared_gpu.json
WORKLOADS="${WORKLOADS:-C1 C2 C3 C4 NS C5 W16K W64K W256K NS_R8 C4_V600 NS_V512}" NCU_WORKLOADS="${NCU_WORKLOADS:-NS C4 C3 C5 W16K W64K}" bash tools/profile_round.sh
