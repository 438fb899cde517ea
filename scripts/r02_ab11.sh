#!/bin/bash
o=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "fuzz or six_vertex or c4_shaped or walker or lane or seven or c3_shaped or symmetry or pipelined" > $o/pytest_ab11.txt 2>&1; echo "pytest exit $?" >> $o/pytest_ab11.txt
GCSM_TRACE=1 timeout 900 python bench.py --quick --steps 2 --warmup 1 --parity-edges 0 > $o/c4_trace8.json 2> $o/c4_trace8.err
out=$o/ab11.txt; : > $out
run() {
  local lab=$1 cfg=$2; shift 2
  env "$@" timeout 900 python bench.py --config $cfg --quick --steps 8 --warmup 3 --parity-edges 0 2>>$o/ab11.err | tail -1 | \
    python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$cfg $lab', round(d['value']), round(d['ms_per_step'],2), {q: (round(x['ms_extend'],2), round(x['ms_walks'],2), x['added'], x['removed']) for q,x in d['per_query'].items()})" >> $out
}
for r in 1 2; do
run def C4 X=1
run ov5 C4 GCSM_OVERLAP_KMAX=5
done
run def C3 X=1
