#!/bin/bash
o=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "fuzz or six_vertex or c4_shaped or walker or seven or c3_shaped or symmetry or full_size_sampled" > $o/pytest_ab12.txt 2>&1; echo "pytest exit $?" >> $o/pytest_ab12.txt
GCSM_TRACE=1 timeout 900 python bench.py --quick --steps 2 --warmup 1 --parity-edges 0 > $o/c4_trace9.json 2> $o/c4_trace9.err
out=$o/ab12.txt; : > $out
run() {
  local lab=$1 cfg=$2; shift 2
  env "$@" timeout 900 python bench.py --config $cfg --quick --steps 8 --warmup 3 --parity-edges 0 2>>$o/ab12.err | tail -1 | \
    python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$cfg $lab', round(d['value']), round(d['ms_per_step'],2), {q: (round(x['ms_extend'],2), round(x['ms_walks'],2), x['added'], x['removed']) for q,x in d['per_query'].items()})" >> $out
}
run def C4 X=1
run def C4 X=1
run def C3 X=1
run ov5 C3 GCSM_OVERLAP_KMAX=5
run def C3 X=1
