#!/bin/bash
# parity tests + a quick bench (no clocks / cpu baseline); used during development
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -p no:cacheprovider > gpurun_out/gpu_tests.txt 2>&1
tail -3 gpurun_out/gpu_tests.txt
timeout 600 python bench.py --quick ${BENCH_ARGS} > gpurun_out/bench_quick.json 2> gpurun_out/bench_quick.err
tail -3 gpurun_out/bench_quick.err
