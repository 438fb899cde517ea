#!/bin/bash
# Paper-style ablations on our kernels: ZP (pure zero-copy), Naive (degree-ranked cache),
# the estimator at several budgets, and all-in-HBM (every list cached: the VSGM-like upper bound).
out=gpurun_out/ablations.jsonl; : > $out
run() { label=$1; shift
  timeout 600 python bench.py --quick --steps 8 --warmup 3 "$@" > gpurun_out/abl.json 2>> gpurun_out/abl.err
  python -c "
import json,sys; d=json.load(open('gpurun_out/abl.json'))
r={'label':'$label','args':'$*','value':d['value'],'ms_per_step':d['ms_per_step'],'cache_hit_rate':d['cache_hit_rate'],
   'per_query':{q:{k:x[k] for k in ('ms_match','ms_extend','hit_rate','cache_mb','miss_gb','host_copied_gb')} for q,x in d['per_query'].items()}}
print(json.dumps(r))" >> $out
}
run estimator_10pct --cache-policy estimator
run zp_budget0 --cache-policy none
run naive_degree_10pct --cache-policy degree
run estimator_1pct --cache-policy estimator --budget-frac 0.01
run estimator_100pct --cache-policy estimator --budget-frac 1.0
run all_in_hbm --cache-policy degree --budget-frac 1.05
# the paper's placement of steps 2-3 (host walks + host packer) for comparison with the GPU estimator/packer
GCSM_HOST_EST=1 run host_estimator_10pct --cache-policy estimator
cat $out
