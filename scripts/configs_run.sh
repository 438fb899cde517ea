#!/bin/bash
# C3 and C4 bench lines (quick: no clocks / cpu baseline), per-query breakdown
timeout 900 python bench.py --quick --config C3 --steps 4 --warmup 2 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; tail -2 gpurun_out/bench_c3.err
timeout 1500 python bench.py --quick --config C4 --steps 3 --warmup 1 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err; tail -2 gpurun_out/bench_c4.err
