#!/bin/bash
# Same-box A/B on C4: the cache step of batch t+1 beside the matching of batch t (default now) vs serial
out=gpurun_out/ab_c4_overlap.txt; : > $out
for v in 8 5 8; do
  GCSM_OVERLAP_KMAX=$v timeout 900 python bench.py --quick --steps 8 --warmup 3 --parity-edges 0 2>/dev/null | tail -1 | \
    python -c "import sys,json; d=json.loads(sys.stdin.read()); print('overlap_kmax=$v', round(d['value']), round(d['ms_per_step'],1), {q: (round(x['ms_extend'],1), round(x['ms_walks'],1)) for q,x in d['per_query'].items()})" >> $out
done
