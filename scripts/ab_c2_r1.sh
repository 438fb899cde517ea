#!/bin/bash
# Same-box A/B of the C2 bench: the round-1 tree (r1tree/, git worktree of dc5db90) against the current build,
# interleaved, quick mode (no clocks / cpu baseline), 16 timed steps each.
out=gpurun_out/ab_c2_r1.txt; : > $out
for i in 1 2; do
  (cd r1tree && timeout 600 python bench.py --config C2 --steps 16 --warmup 4 --quick 2>/dev/null | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('r1', d['value'], d['ms_per_step'])") >> $out
  timeout 600 python bench.py --config C2 --steps 16 --warmup 4 --quick --parity-edges 0 2>/dev/null | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('r2', d['value'], d['ms_per_step'])" >> $out
done
