#!/bin/bash
# Same-box A/B of environment switches / variant libraries on one bench config (one GPU):
#   bash scripts/ab_env.sh C4 8 "def:X=1" "nofsplit:GCSM_NO_FSPLIT=1" "mb2:GCSM_LIB=variants/libgcsm_mb2.so"
# Each arm runs twice, interleaved; one line per run in gpurun_out/ab_env.txt (value, ms per step, per query:
# extension ms, walk ms, added, removed).
cfg=$1; steps=$2; shift 2
o=gpurun_out; out=$o/ab_env.txt; : > $out
for r in 1 2; do
  for arm in "$@"; do
    lab=${arm%%:*}; envs=${arm#*:}
    env ${envs//,/ } timeout 900 python bench.py --config $cfg --quick --steps $steps --warmup 3 --parity-edges 0 2>>$o/ab_env.err | tail -1 | \
      python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$cfg $lab', round(d['value']), round(d['ms_per_step'],2), {q: (round(x['ms_extend'],2), round(x['ms_walks'],2), x['added'], x['removed']) for q,x in d['per_query'].items()})" >> $out
  done
done
