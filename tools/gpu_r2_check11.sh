# Early row prefetch: A/B (PSO_EARLY=0/1) on C3, NS, C4, NS_R8 (+ forced exchange), then parity tests.
exec > gpurun_out/check11.log 2>&1
for e in 1 0 1 0; do echo "== PSO_EARLY=$e"; PSO_EARLY=$e WORKLOADS="C3 NS_R8 C4 NS" STEPS=500 bash tools/bench_sweep.sh; done
for e in 1 0; do echo "== PSO_EARLY=$e forced exchange NS_R8"; PSO_EARLY=$e PSO_FORCE_EXCHANGE=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29517 bench.py --workload NS_R8 --steps 1000 --warmup 20 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys
j=json.loads(sys.stdin.read()); r=j['roofline']
print(f\"{j['ms_per_step']*1e3:8.2f} us/step kern {r['kernel_avg_us']:8.2f} us {j['config'].get('gbest_exchange')} clk {j['clocks']['sm_mhz']}\")"; done
timeout 2400 python -m pytest tests -m gpu -q -x 2>&1 | tail -8
