#!/bin/bash
# Final check of the committed state: build, GPU tests, smoke, one default bench line. Usage: bash scripts/final_check.sh <tag>
T=${1:-final}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$T.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/pytest_gpu_$T.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_$T.txt 2>&1
timeout 900 python bench.py > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err
tail -1 gpurun_out/pytest_gpu_$T.txt; tail -1 gpurun_out/smoke_$T.txt; tail -1 gpurun_out/bench_$T.json | cut -c1-200
