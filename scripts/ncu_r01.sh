#!/bin/bash
# ncu evidence for round 1 (run under gpurun). Launch list (cold, serialised) + full captures of the top kernels.
set -x
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01.csv \
    python bench.py --steps 2 --warmup 1 --quick > gpurun_out/ncu_launch_bench.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_extend -s 1 -c 1 -o gpurun_out/prof_extend_c4 -f \
    python bench.py --steps 1 --warmup 1 --quick --queries c4 > gpurun_out/ncu_full_c4.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_extend -s 1 -c 1 -o gpurun_out/prof_extend_k4 -f \
    python bench.py --steps 1 --warmup 1 --quick --queries k4 > gpurun_out/ncu_full_k4.txt 2>&1
ncu --query-metrics > gpurun_out/ncu_metrics_list.txt 2>&1
