#!/bin/bash
# dev: kernel counters (GCSM_TRACE) + full ncu capture (source-attributed) of the c4 last-level launch; tag in $1
T=${1:-dev}
GCSM_TRACE=1 timeout 300 python bench.py --quick --serial --steps 3 --warmup 2 --queries c4 > gpurun_out/tr_c4_$T.json 2> gpurun_out/tr_c4_$T.err
grep "gcsm kern" gpurun_out/tr_c4_$T.err | tail -3
ncu --set full --clock-control none --import-source on -k regex:"k_extend|k_last4" -s 1 -c 1 -o gpurun_out/prof_ext_c4_$T -f \
    python bench.py --steps 1 --warmup 1 --quick --queries c4 ${NCU_BENCH_ARGS} > gpurun_out/ncu_c4_$T.txt 2>&1
ncu -i gpurun_out/prof_ext_c4_$T.ncu-rep --page source --csv --print-source sass > gpurun_out/src_c4_$T.csv 2>&1
ncu -i gpurun_out/prof_ext_c4_$T.ncu-rep --page raw --csv > gpurun_out/raw_c4_$T.csv 2>&1
