#!/bin/bash
# Cache step of batch t+1 beside batch t's matching (stream3) vs on the context stream (GCSM_NO_OVERLAP=1):
# GPU tests with the overlap on, then alternating C2 / C3 bench --quick runs, then the default C2 bench line.
# Usage (under gpurun): bash scripts/ab_overlap.sh <tag>
T=${1:-dev}
out=gpurun_out/ab_overlap_$T.txt; : > $out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$T.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/pytest_gpu_$T.txt 2>&1
echo "tests: $(tail -1 gpurun_out/pytest_gpu_$T.txt)" >> $out
for cfg in C2 C3; do for rep in 1 2; do for v in on off; do
  if [ $v = off ]; then export GCSM_NO_OVERLAP=1; else unset GCSM_NO_OVERLAP; fi
  timeout 600 python bench.py --quick --config $cfg > gpurun_out/abo_${cfg}_$v.json 2>>gpurun_out/abo.err
  python -c "
import json; d=json.loads(open('gpurun_out/abo_${cfg}_$v.json').read().strip().splitlines()[-1])
print('$cfg', '$v', $rep, round(d['value']), round(d['ms_per_step'],2), {q: ('match', round(x['ms_match'],2), 'copy', round(x['breakdown_ms']['ms_copy'],2), 'host_gb', round(x['host_copied_gb'],3)) for q,x in d['per_query'].items()})" >> $out
done; done; done
unset GCSM_NO_OVERLAP
timeout 900 python bench.py > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err
cat $out
