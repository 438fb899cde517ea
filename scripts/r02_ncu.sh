#!/bin/bash
# ncu captures (one GPU, after the plain runs exited 0): C4 prism6 k_walks + k_extend of batch 1, C2 c4 k_last4.
o=gpurun_out
NCU=/usr/local/cuda/bin/ncu
NB=2 QUERIES=prism6 timeout 900 python scripts/c4_ncu.py > $o/c4_plain.txt 2>&1; echo "plain exit $?" >> $o/c4_plain.txt
NB=2 QUERIES=prism6 timeout 1500 $NCU --set full --import-source on --clock-control none --kernel-name-base function \
  -k regex:"^(k_extend|k_walks)$" --launch-skip 2 --launch-count 2 -f -o $o/ncu_c4_prism6_r02 \
  python scripts/c4_ncu.py > $o/ncu_c4.log 2>&1; echo "ncu exit $?" >> $o/ncu_c4.log
CFG=C2 NB=5 QUERIES=c4 timeout 900 $NCU --set full --import-source on --clock-control none --kernel-name-base function \
  -k regex:"^k_last4$" --launch-skip 3 --launch-count 1 -f -o $o/ncu_c2_last4_r02 \
  python scripts/c4_ncu.py > $o/ncu_c2.log 2>&1; echo "ncu exit $?" >> $o/ncu_c2.log
