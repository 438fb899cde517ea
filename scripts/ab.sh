#!/bin/bash
# A/B kernel variants (serial, match-only numbers; C2 K4+C4 in one context): VARIANTS="a b" [ARGSETS as below]
out=gpurun_out/ab.txt; : > $out
for args in "--cache-policy estimator" "--cache-policy degree --budget-frac 1.05"; do
for v in ${VARIANTS:-old new}; do
  GCSM_LIB=$PWD/variants/libgcsm_$v.so timeout 300 python bench.py --quick --serial --steps 4 --warmup 2 $args > gpurun_out/ab_$v.json 2>>gpurun_out/ab.err
  python -c "
import json; d=json.load(open('gpurun_out/ab_$v.json'))
print('$v', '$args', round(d['value']), {q: dict(match=round(x['ms_match'],3), ext=round(x['ms_extend'],3), l2=round(x['ms_level2'],3), copied=round(x['host_copied_gb'],3)) for q,x in d['per_query'].items()})" >> $out
done; done
cat $out
