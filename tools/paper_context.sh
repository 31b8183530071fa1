exec > gpurun_out/context.log 2>&1
python tools/paper_table1.py > gpurun_out/paper_table1.txt 2>&1
cat gpurun_out/paper_table1.txt
bash tools/oracle_sweep.sh > gpurun_out/oracle_full.jsonl 2>&1
cat gpurun_out/oracle_full.jsonl
for w in C1 C2 C3 C4 NS C5; do python -c "
import json; j=json.load(open('gpurun_out/oracle_$w.json')); print('$w', j['value'], j['cpu_baseline']['sample'])"; done
