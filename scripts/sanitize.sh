#!/bin/bash
# compute-sanitizer memcheck on a subset of the GPU parity tests (small inputs); writes gpurun_out/sanitizer_*.txt
export PYTHONUNBUFFERED=1
timeout 1500 compute-sanitizer --tool memcheck --leak-check no --error-exitcode 9 \
  python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider \
  -k "c1_triangle or fuzz_small_graphs or degenerate or stream_of_mixed or six_vertex or pipelined or interleaved or c3_shaped or estimator or budget_change or degree_policy" \
  > gpurun_out/sanitizer_memcheck.txt 2>&1
echo "memcheck rc=$?" >> gpurun_out/sanitizer_memcheck.txt
tail -5 gpurun_out/sanitizer_memcheck.txt
timeout 1500 compute-sanitizer --tool racecheck --error-exitcode 9 \
  python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider \
  -k "c1_triangle or fuzz_small_graphs or six_vertex or c3_shaped or estimator_and_cache" > gpurun_out/sanitizer_racecheck.txt 2>&1
echo "racecheck rc=$?" >> gpurun_out/sanitizer_racecheck.txt
tail -5 gpurun_out/sanitizer_racecheck.txt
timeout 1500 compute-sanitizer --tool synccheck --error-exitcode 9 \
  python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider \
  -k "c1_triangle or fuzz_small_graphs or six_vertex" > gpurun_out/sanitizer_synccheck.txt 2>&1
echo "synccheck rc=$?" >> gpurun_out/sanitizer_synccheck.txt
tail -5 gpurun_out/sanitizer_synccheck.txt
