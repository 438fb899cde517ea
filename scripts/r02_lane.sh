#!/bin/bash
# Lane-parallel level k-3 walk nodes: product-internal equality tests, then a same-box C4 A/B.
o=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "walker or lane or eq6 or six_vertex or c4_shaped" > $o/pytest_lane.txt 2>&1; echo "pytest exit $?" >> $o/pytest_lane.txt
out=$o/ab_walk_lane.txt; : > $out
for v in 1 0 1; do
  GCSM_WALK_LANE=$v timeout 900 python bench.py --quick --steps 8 --warmup 3 --parity-edges 0 2>>$o/ab_walk_lane.err | tail -1 | \
    python -c "import sys,json; d=json.loads(sys.stdin.read()); print('walk_lane=$v', round(d['value']), round(d['ms_per_step'],1), {q: (round(x['ms_extend'],1), round(x['ms_walks'],1), x['added'], x['removed']) for q,x in d['per_query'].items()})" >> $out
done
bash scripts/r02_shared.sh
