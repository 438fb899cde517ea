#!/bin/bash
# GPU estimator dev cycle: parity tests, quick bench, serial ncu launch list, traced run
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -p no:cacheprovider > gpurun_out/gpu_tests.txt 2>&1; tail -3 gpurun_out/gpu_tests.txt
timeout 600 python bench.py --quick ${BENCH_ARGS} > gpurun_out/bq.json 2> gpurun_out/bq.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_est.csv python bench.py --steps 2 --warmup 1 --quick --serial ${BENCH_ARGS} > gpurun_out/ncu_launch_est.txt 2>&1
GCSM_TRACE=1 timeout 300 python bench.py --quick --steps 4 --warmup 2 ${BENCH_ARGS} > gpurun_out/tr.json 2> gpurun_out/tr.err
