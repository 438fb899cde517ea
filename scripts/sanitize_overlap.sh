#!/bin/bash
# compute-sanitizer memcheck on the pipelined (two in flight, cache step on its own stream) small-graph tests
export PYTHONUNBUFFERED=1
timeout 900 compute-sanitizer --tool memcheck --leak-check no --error-exitcode 9 \
  python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider \
  -k "pipelined_submit or multi_query or c1_triangle or budget_change" > gpurun_out/sanitizer_memcheck_overlap.txt 2>&1
echo "memcheck rc=$?" >> gpurun_out/sanitizer_memcheck_overlap.txt
tail -3 gpurun_out/sanitizer_memcheck_overlap.txt
