#!/bin/bash
# time tuning variants of libgcsm on the bench (quick mode)
for v in ${VARIANTS:-A B C D E}; do
  GCSM_LIB=$PWD/variants/libgcsm_$v.so timeout 300 python bench.py --quick --steps 4 --warmup 2 ${BENCH_ARGS} > gpurun_out/var_$v.json 2>gpurun_out/var_$v.err
  python -c "
import json; d=json.load(open('gpurun_out/var_$v.json'))
print('$v', round(d['value']), {q: (round(x['ms_match'],2), round(x['ms_per_batch'],2)) for q,x in d['per_query'].items()})"
done
