bash scripts/trace_c2.sh
out=gpurun_out/abl1.jsonl; : > $out
for a in "--cache-policy estimator" "--cache-policy degree --budget-frac 1.05"; do
timeout 600 python bench.py --quick --serial --steps 4 --warmup 2 $a > gpurun_out/abl.json 2>> gpurun_out/abl.err
python -c "
import json,sys; d=json.load(open('gpurun_out/abl.json'))
r={'args':'$a','value':d['value'],'ms_per_step':d['ms_per_step'],
   'per_query':{q:{k:x[k] for k in ('ms_match','ms_extend','ms_level2','hit_rate','cache_mb','miss_gb','host_copied_gb','frontier','breakdown_ms')} for q,x in d['per_query'].items()}}
print(json.dumps(r))" >> $out
done
