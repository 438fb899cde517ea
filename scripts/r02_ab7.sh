#!/bin/bash
o=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "fuzz or six_vertex or c4_shaped or walker or lane or seven or c3_shaped or symmetry or full_size_sampled" > $o/pytest_ab7.txt 2>&1; echo "pytest exit $?" >> $o/pytest_ab7.txt
GCSM_TRACE=1 timeout 900 python bench.py --quick --steps 2 --warmup 1 --parity-edges 0 > $o/c4_trace4.json 2> $o/c4_trace4.err
out=$o/ab7.txt; : > $out
for cfg in C4 C3 C2; do
for v in def mb2 def mb2; do
  lib=""; [ $v == mb2 ] && lib=variants/libgcsm_mb2.so
  GCSM_LIB=$lib timeout 900 python bench.py --config $cfg --quick --steps 8 --warmup 3 --parity-edges 0 2>>$o/ab7.err | tail -1 | \
    python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$cfg $v', round(d['value']), round(d['ms_per_step'],2), {q: (round(x['ms_extend'],2), round(x['ms_walks'],2), x['added'], x['removed']) for q,x in d['per_query'].items()})" >> $out
done; done
