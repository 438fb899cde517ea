#!/bin/bash
o=gpurun_out
out=$o/ab14.txt; : > $out
for v in def deep def deep; do
  lib=""; [ $v == deep ] && lib=variants/libgcsm_deep.so
  GCSM_LIB=$lib timeout 900 python bench.py --quick --steps 8 --warmup 3 --parity-edges 0 2>>$o/ab14.err | tail -1 | \
    python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$v', round(d['value']), round(d['ms_per_step'],2), {q: (round(x['ms_extend'],2), round(x['ms_walks'],2), x['added'], x['removed']) for q,x in d['per_query'].items()})" >> $out
done
