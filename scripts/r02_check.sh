#!/bin/bash
# Round-2 state check on one B200: GPU tests, smoke, the default bench (C4) and C2.
o=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $o/gpu.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider --durations=25 > $o/pytest_gpu.txt 2>&1; echo "pytest exit $?" >> $o/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $o/smoke.txt 2>&1; echo "smoke exit $?" >> $o/smoke.txt
timeout 1200 python bench.py > $o/bench_c4.json 2> $o/bench_c4.err; echo "bench exit $?" >> $o/bench_c4.err
timeout 600 python bench.py --config C2 > $o/bench_c2.json 2> $o/bench_c2.err; echo "bench exit $?" >> $o/bench_c2.err
