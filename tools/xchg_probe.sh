L="python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29517"
for fx in 0 1; do
  PSO_FORCE_EXCHANGE=$fx timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_step -c 60 --csv --log-file gpurun_out/xl_$fx.csv $L bench.py --workload NS_R8 --steps 40 --warmup 5 --no-e2e --no-cpu-baseline > /dev/null 2>&1
done
for fx in 0 1; do for pdl in 1 0; do
  PSO_PDL=$pdl PSO_FORCE_EXCHANGE=$fx timeout 300 $L bench.py --workload NS_R8 --steps 500 --warmup 10 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys
j=json.loads(sys.stdin.read()); r=j['roofline']
print('xchg=$fx pdl=$pdl', f\"{j['ms_per_step']*1e3:8.2f} us/step kern {r['kernel_avg_us']:8.2f}\")"
done; done
