#!/bin/bash
# A/B of the sampled-index stride (and k_last4 occupancy): parity of the C2-shaped and full-size sampled tests with
# each variant, then alternating C2 bench --quick runs. Usage (under gpurun): bash scripts/ab_sidx.sh
out=gpurun_out/ab_sidx2.txt; : > $out
for v in ${VARIANTS:-s32 s16 s8}; do
  GCSM_LIB=$PWD/variants/libgcsm_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x \
    -k "c2_shaped or full_size_sampled" -p no:cacheprovider > gpurun_out/ab_sidx_tests_$v.txt 2>&1
  echo "$v tests: $(tail -1 gpurun_out/ab_sidx_tests_$v.txt)" >> $out
done
for rep in 1 2; do for v in ${VARIANTS:-s32 s16 s8}; do
  GCSM_LIB=$PWD/variants/libgcsm_$v.so timeout 300 python bench.py --quick > gpurun_out/ab_sidx_$v.json 2>>gpurun_out/ab_sidx.err
  python -c "
import json; d=json.load(open('gpurun_out/ab_sidx_$v.json'))
print('$v', $rep, round(d['value']), round(d['ms_per_step'],2), {q: ('match_ms', round(x['ms_match'],2), 'host_gb', round(x['host_copied_gb'],3)) for q,x in d['per_query'].items()})" >> $out
done; done
cat $out
