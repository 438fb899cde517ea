#!/bin/bash
GCSM_TRACE=1 timeout 600 python bench.py --quick --steps 4 --warmup 2 ${BENCH_ARGS} > gpurun_out/trace.json 2> gpurun_out/trace.err
grep "gcsm trace" gpurun_out/trace.err | tail -8
