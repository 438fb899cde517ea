#!/bin/bash
# dev cycle: GPU parity tests, a quick bench, one traced run (host sub-steps + kernel counters)
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -p no:cacheprovider > gpurun_out/gpu_tests.txt 2>&1; tail -3 gpurun_out/gpu_tests.txt
timeout 600 python bench.py --quick ${BENCH_ARGS} > gpurun_out/bench_quick.json 2> gpurun_out/bench_quick.err; tail -3 gpurun_out/bench_quick.err
GCSM_TRACE=1 timeout 300 python bench.py --quick --steps 4 --warmup 2 > gpurun_out/tr.json 2> gpurun_out/tr.err; grep "gcsm" gpurun_out/tr.err | tail -6
