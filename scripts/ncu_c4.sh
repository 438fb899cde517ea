#!/bin/bash
T=${1:-dev}
ncu --set full --clock-control none --import-source on -k regex:k_extend -s 1 -c 1 -o gpurun_out/prof_ext_c4_$T -f \
    python bench.py --steps 1 --warmup 1 --quick --queries c4 > gpurun_out/ncu_c4_$T.txt 2>&1
