# Per-rank step time of the NS shards at 2/4/8 GPUs, on one GPU: kernel only,
# then with the exchange path forced (1-rank process group, NVLink-peer records).
for w in ${WORKLOADS:-NS NS_R2 NS_R4 NS_R8}; do
  for fx in 0 1; do
    if [ $fx = 1 ]; then
      L="python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29517"
    else
      L=python
    fi
    PSO_FORCE_EXCHANGE=$fx timeout 300 $L bench.py --workload $w --steps ${STEPS:-500} --warmup 10 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys
j=json.loads(sys.stdin.read()); r=j['roofline']
print('$w xchg=$fx', f\"{j['ms_per_step']*1e3:8.2f} us/step kern {r['kernel_avg_us']:8.2f} us frac {r['frac']:.3f} {j['config'].get('gbest_exchange')} launches {j['gpu_launches']} clk {j['clocks']['sm_mhz']}\")" || echo "$w $fx FAILED"
  done
done
