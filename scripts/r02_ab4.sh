#!/bin/bash
o=gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "fuzz or six_vertex or c4_shaped or walker or lane or seven or c2_shaped or c3_shaped or pipelined" > $o/pytest_ab4.txt 2>&1; echo "pytest exit $?" >> $o/pytest_ab4.txt
out=$o/ab_minblocks.txt; : > $out
for v in base mb3 mb2 base mb3 mb2; do
  lib=""; [ $v != base ] && lib=variants/libgcsm_$v.so
  GCSM_LIB=$lib timeout 900 python bench.py --quick --steps 6 --warmup 2 --parity-edges 0 2>>$o/ab_minblocks.err | tail -1 | \
    python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$v', round(d['value']), round(d['ms_per_step'],1), {q: (round(x['ms_extend'],1), round(x['ms_walks'],1), round(x['ms_level2'],1)) for q,x in d['per_query'].items()})" >> $out
done
