#!/bin/bash
# Round evidence (GPU estimator era): full bench line (C2 default), ncu launch list (cold, serialised), full captures
# of the top kernel (c4's k_last4), the GPU walks (k_walks_l1) and cache copy (k_copy), and C3 K5-e's k_extend.
# Usage (under gpurun): bash scripts/evidence2.sh <tag>
T=${1:-dev}
timeout 900 python bench.py > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$T.csv \
    python bench.py --steps 2 --warmup 1 --quick --serial > gpurun_out/ncu_launch_$T.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_last4" -s 1 -c 1 -o gpurun_out/prof_c4_$T -f \
    python bench.py --steps 1 --warmup 1 --quick --serial --queries c4 > gpurun_out/ncu_c4_$T.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_walks_l1|k_copy" -s 2 -c 2 -o gpurun_out/prof_est_$T -f \
    python bench.py --steps 1 --warmup 1 --quick --serial > gpurun_out/ncu_est_$T.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_extend" -s 1 -c 1 -o gpurun_out/prof_k5e_$T -f \
    python bench.py --config C3 --steps 1 --warmup 1 --quick --serial --queries k5e > gpurun_out/ncu_k5e_$T.txt 2>&1
