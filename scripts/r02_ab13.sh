#!/bin/bash
o=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "fuzz or six_vertex or c4_shaped or seven or symmetry or full_size_c4" > $o/pytest_ab13.txt 2>&1; echo "pytest exit $?" >> $o/pytest_ab13.txt
GCSM_TRACE=1 timeout 900 python bench.py --quick --steps 2 --warmup 1 --parity-edges 0 > $o/c4_trace10.json 2> $o/c4_trace10.err
out=$o/ab13.txt; : > $out
for r in 1 2 3; do
  timeout 900 python bench.py --quick --steps 8 --warmup 3 --parity-edges 0 2>>$o/ab13.err | tail -1 | \
    python -c "import sys,json; d=json.loads(sys.stdin.read()); print('gallop', round(d['value']), round(d['ms_per_step'],2), {q: (round(x['ms_extend'],2), round(x['ms_walks'],2), x['added'], x['removed']) for q,x in d['per_query'].items()})" >> $out
done
