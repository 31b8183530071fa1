exec > gpurun_out/check10.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q -k "exchange or nvlink or switch or multirank or decisions or empty" 2>&1 | tail -15
for m in nccl allreduce p2p; do echo "== PSO_EXCHANGE=$m NS_R8 forced exchange (1 rank)"; PSO_EXCHANGE=$m PSO_FORCE_EXCHANGE=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29517 bench.py --workload NS_R8 --steps 500 --warmup 10 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys
j=json.loads(sys.stdin.read()); r=j['roofline']
print(f\"{j['ms_per_step']*1e3:8.2f} us/step kern {r['kernel_avg_us']:8.2f} us frac {r['frac']:.3f} {j['config'].get('gbest_exchange')} launches {j['gpu_launches']} clk {j['clocks']['sm_mhz']}\")"; done
echo "== NS_R8 no exchange"; WORKLOADS="NS_R8" STEPS=500 bash tools/bench_sweep.sh
