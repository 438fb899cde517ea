#!/bin/bash
o=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_multiproc.py -m gpu -x -q -p no:cacheprovider -k "lane or walker or shared or world2 or emulated or shard" > $o/pytest_run3.txt 2>&1; echo "pytest exit $?" >> $o/pytest_run3.txt
GCSM_TRACE=1 timeout 900 python bench.py --quick --steps 3 --warmup 2 --parity-edges 0 > $o/c4_trace.json 2> $o/c4_trace.err
for n in 2 4; do
  timeout 900 python bench.py --config C2 --gpus $n --emulate --quick --steps 8 --warmup 3 > $o/emul_C2_n${n}_shared.json 2> $o/emul_C2_n${n}_shared.err
done
bash scripts/r02_ncu.sh
