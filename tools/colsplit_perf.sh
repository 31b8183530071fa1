exec > gpurun_out/check21.log 2>&1
WORKLOADS="W64K W256K" STEPS=200 bash tools/bench_sweep.sh
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_W64K.csv python bench.py --workload W64K --steps 10 --warmup 5 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python - <<'PY'
import csv
from collections import defaultdict
rows=list(csv.reader(open('gpurun_out/launches_W64K.csv')))
hdr=None; data=[]
for r in rows:
    if r and r[0]=='ID': hdr=r; continue
    if hdr and len(r)==len(hdr): data.append(dict(zip(hdr,r)))
tot=defaultdict(list)
for d in data:
    if d.get('Metric Name')=='gpu__time_duration.sum': tot[d['Kernel Name'][:60]].append(float(d['Metric Value']))
for k,v in tot.items(): print(k, len(v), sum(v)/len(v))
PY
timeout 1800 python -m pytest tests -m gpu -q -k "column or colsplit or col_ or maximum" 2>&1 | tail -3
