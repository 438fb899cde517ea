#!/bin/bash
o=gpurun_out
GCSM_TRACE=1 timeout 900 python bench.py --quick --steps 2 --warmup 1 --parity-edges 0 > $o/c4_trace7.json 2> $o/c4_trace7.err
out=$o/ab10.txt; : > $out
run() {
  local lab=$1 cfg=$2; shift 2
  env "$@" timeout 900 python bench.py --config $cfg --quick --steps 8 --warmup 3 --parity-edges 0 2>>$o/ab10.err | tail -1 | \
    python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$cfg $lab', round(d['value']), round(d['ms_per_step'],2), {q: (round(x['ms_extend'],2), round(x['ms_walks'],2), x['added'], x['removed']) for q,x in d['per_query'].items()})" >> $out
}
run def C4 X=1
run overlap8 C4 GCSM_OVERLAP_KMAX=8
run def C4 X=1
run overlap8 C4 GCSM_OVERLAP_KMAX=8
