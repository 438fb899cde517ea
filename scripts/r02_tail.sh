#!/bin/bash
# Late evidence: k_last4 under ncu on the final tree; emulated N = 2 / 4 C2 benches over the shared store with the
# cross-process peer cache linked (every rank on cuda:0).
o=gpurun_out
CFG=C2 NB=5 QUERIES=c4 timeout 900 /usr/local/cuda/bin/ncu --set full --import-source on --clock-control none --kernel-name-base function \
  -k regex:"^k_last4$" --launch-skip 3 --launch-count 1 -f -o $o/ncu_c2_last4_final \
  python scripts/c4_ncu.py > $o/tail_ncu_c2.log 2>&1; echo "exit $?" >> $o/tail_ncu_c2.log
for n in 2 4; do
  timeout 900 python bench.py --config C2 --gpus $n --emulate --quick --steps 8 --warmup 3 > $o/tail_emul_C2_n${n}.json 2> $o/tail_emul_C2_n${n}.err
done
