#!/bin/bash
o=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "fuzz or six_vertex or c4_shaped or walker or lane or seven or c3_shaped or eq6 or symmetry" > $o/pytest_ab6.txt 2>&1; echo "pytest exit $?" >> $o/pytest_ab6.txt
GCSM_TRACE=1 timeout 900 python bench.py --quick --steps 2 --warmup 1 --parity-edges 0 > $o/c4_trace3.json 2> $o/c4_trace3.err
out=$o/ab_fsplit.txt; : > $out
for v in def nofs mb2 def nofs mb2; do
  lib=""; [ $v == mb2 ] && lib=variants/libgcsm_mb2.so
  nf=""; [ $v == nofs ] && nf=1
  env ${nf:+GCSM_NO_FSPLIT=1} GCSM_LIB=$lib timeout 900 python bench.py --quick --steps 6 --warmup 2 --parity-edges 0 2>>$o/ab_fsplit.err | tail -1 | \
    python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$v', round(d['value']), round(d['ms_per_step'],1), {q: (round(x['ms_extend'],1), round(x['ms_walks'],1), x['added'], x['removed']) for q,x in d['per_query'].items()})" >> $out
done
