# Exchange-latency experiment on the 1-rank proxy (NS_R8 with the NVLink exchange forced).
# Round 2 measured the record tag's system-scope release by building once with a relaxed store
# in its place (-DPSO_EXP_RELAXED_TAG around st_release_sys_u64 in epilogue_core); that
# experiment-only switch is not kept in the kernels (it has no ordering guarantee), so the
# second pair of runs below now repeats the baseline unless it is re-added.
exec > gpurun_out/exp1.log 2>&1
run() { PSO_FORCE_EXCHANGE=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29517 bench.py --workload NS_R8 --steps 1000 --warmup 20 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys
j=json.loads(sys.stdin.read()); r=j['roofline']
print(f\"$1: {j['ms_per_step']*1e3:8.2f} us/step kern {r['kernel_avg_us']:8.2f} us {j['config'].get('gbest_exchange')} clk {j['clocks']['sm_mhz']}\")"; }
run baseline; run baseline2
make lib -j16 EXTRA=-DPSO_EXP_RELAXED_TAG -B > /dev/null 2>&1 && run relaxed_tag && run relaxed_tag2
WORKLOADS="NS_R8" STEPS=1000 bash tools/bench_sweep.sh
