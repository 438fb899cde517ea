#!/bin/bash
# Extension-kernel blocks left free for the overlapped cache step (GCSM_EXT_RESERVE) and the cache stream's
# priority (GCSM_CS_PRIO): C2 bench --quick, alternating twice on one box. Usage (under gpurun): bash scripts/ab_reserve.sh
out=gpurun_out/ab_reserve.txt; : > $out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rep in 1 2; do for v in "r0" "r0p" "r24" "r24p" "r74p" "r148p"; do
  unset GCSM_CS_PRIO; r=${v#r}; r=${r%p}; [ "${v: -1}" = p ] && export GCSM_CS_PRIO=1
  GCSM_EXT_RESERVE=$r timeout 300 python bench.py --quick > gpurun_out/abr_$v.json 2>>gpurun_out/abr.err
  python -c "
import json; d=json.loads(open('gpurun_out/abr_$v.json').read().strip().splitlines()[-1])
print('$v', $rep, round(d['value']), round(d['ms_per_step'],2), {q: ('match', round(x['ms_match'],2), 'copy', round(x['breakdown_ms']['ms_copy'],2)) for q,x in d['per_query'].items()})" >> $out
done; done
cat $out
