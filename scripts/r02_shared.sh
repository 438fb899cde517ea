#!/bin/bash
# Node-shared host store on one B200: the multi-process GPU tests, then emulated N = 1/2/4 benches (every rank on
# cuda:0, gloo) with the shared store and with private replicas, recording per-rank host time and memory.
o=gpurun_out
timeout 900 python -m pytest tests/test_multiproc.py -m gpu -x -q -p no:cacheprovider > $o/pytest_shared.txt 2>&1; echo "pytest exit $?" >> $o/pytest_shared.txt
for cfg in C2; do
  timeout 600 python bench.py --config $cfg --quick --steps 8 --warmup 3 > $o/emul_${cfg}_n1.json 2> $o/emul_${cfg}_n1.err
  for n in 2 4; do
    timeout 900 python bench.py --config $cfg --gpus $n --emulate --quick --steps 8 --warmup 3 > $o/emul_${cfg}_n${n}_shared.json 2> $o/emul_${cfg}_n${n}_shared.err
    timeout 900 python bench.py --config $cfg --gpus $n --emulate --quick --steps 8 --warmup 3 --private-store > $o/emul_${cfg}_n${n}_private.json 2> $o/emul_${cfg}_n${n}_private.err
  done
done
