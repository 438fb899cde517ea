#!/bin/bash
# Round evidence v15 (overlapped cache step, default build) then k_last4 occupancy / merge variants A/B.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_r01_v15.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/pytest_gpu_r01_v15.txt 2>&1
bash scripts/evidence3.sh r01_v15
out=gpurun_out/ab_l4var.txt; : > $out
for v in m4 mi4 m2; do
  GCSM_LIB=$PWD/variants/libgcsm_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x \
    -k "c2_shaped or full_size_sampled" -p no:cacheprovider > gpurun_out/ab_l4var_tests_$v.txt 2>&1
  echo "$v tests: $(tail -1 gpurun_out/ab_l4var_tests_$v.txt)" >> $out
done
for rep in 1 2; do for v in base m4 mi4 m2; do
  GCSM_LIB=$PWD/variants/libgcsm_$v.so timeout 300 python bench.py --quick > gpurun_out/abv_$v.json 2>>gpurun_out/abv.err
  python -c "
import json; d=json.loads(open('gpurun_out/abv_$v.json').read().strip().splitlines()[-1])
print('$v', $rep, round(d['value']), round(d['ms_per_step'],2), {q: ('match', round(x['ms_match'],2), 'ext', round(x['ms_extend'],2)) for q,x in d['per_query'].items()})" >> $out
done; done
cat $out
