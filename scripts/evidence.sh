#!/bin/bash
# Round evidence: full bench line, ncu launch list (cold, serialised), full capture of the top kernel (c4 k_extend)
# and of k4's k_extend, k_level2. Usage (under gpurun): bash scripts/evidence.sh <tag>
T=${1:-dev}
timeout 900 python bench.py > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$T.csv \
    python bench.py --steps 2 --warmup 1 --quick --serial > gpurun_out/ncu_launch_$T.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_extend -s 1 -c 1 -o gpurun_out/prof_ext_c4_$T -f \
    python bench.py --steps 1 --warmup 1 --quick --serial --queries c4 > gpurun_out/ncu_c4_$T.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_extend|k_level2" -s 2 -c 2 -o gpurun_out/prof_k4_$T -f \
    python bench.py --steps 1 --warmup 1 --quick --serial --queries k4 > gpurun_out/ncu_k4_$T.txt 2>&1
