#!/bin/bash
o=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_multiproc.py -m gpu -x -q -p no:cacheprovider -k "fuzz or six_vertex or c4_shaped or walker or lane or seven or c2_shaped or c3_shaped or pipelined or eq6 or shared or peer" > $o/pytest_ab5.txt 2>&1; echo "pytest exit $?" >> $o/pytest_ab5.txt
out=$o/ab_lane_root.txt; : > $out
for v in lane nolane mb2 lane nolane mb2; do
  lib=""; [ $v == mb2 ] && lib=variants/libgcsm_mb2.so
  wl=1; [ $v == nolane ] && wl=0
  GCSM_WALK_LANE=$wl GCSM_LIB=$lib timeout 900 python bench.py --quick --steps 6 --warmup 2 --parity-edges 0 2>>$o/ab_lane_root.err | tail -1 | \
    python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$v', round(d['value']), round(d['ms_per_step'],1), {q: (round(x['ms_extend'],1), round(x['ms_walks'],1), x['added'], x['removed']) for q,x in d['per_query'].items()})" >> $out
done
GCSM_TRACE=1 timeout 900 python bench.py --quick --steps 2 --warmup 1 --parity-edges 0 > /dev/null 2> $o/c4_trace2.err
