#!/bin/bash
# Round evidence: full bench line (C2 default), ncu launch list (cold, serialised), full captures of the top
# kernel (c4's last-level kernel) and of k4's level-2 + last-level kernels. Usage (under gpurun): bash scripts/evidence.sh <tag>
T=${1:-dev}
timeout 900 python bench.py > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$T.csv \
    python bench.py --steps 2 --warmup 1 --quick --serial > gpurun_out/ncu_launch_$T.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_extend|k_last4" -s 1 -c 1 -o gpurun_out/prof_ext_c4_$T -f \
    python bench.py --steps 1 --warmup 1 --quick --serial --queries c4 > gpurun_out/ncu_c4_$T.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_extend|k_last4|k_level2" -s 2 -c 2 -o gpurun_out/prof_k4_$T -f \
    python bench.py --steps 1 --warmup 1 --quick --serial --queries k4 > gpurun_out/ncu_k4_$T.txt 2>&1
ncu -i gpurun_out/prof_ext_c4_$T.ncu-rep --page source --csv --print-source sass > gpurun_out/src_c4_$T.csv 2>&1
