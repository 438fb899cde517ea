#!/bin/bash
# Round-2 evidence on one B200: GPU tests, smoke, the default bench (C4) and C2 / C3 lines, the reference arm, the
# launch list of the bench command and one full ncu capture of the dominant kernels (prism6 walks + extension).
o=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $o/final_gpu.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider --durations=15 > $o/final_pytest_gpu.txt 2>&1; echo "pytest exit $?" >> $o/final_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $o/final_smoke.txt 2>&1; echo "smoke exit $?" >> $o/final_smoke.txt
timeout 1200 python bench.py > $o/final_bench_c4.json 2> $o/final_bench_c4.err; echo "exit $?" >> $o/final_bench_c4.err
timeout 900 python bench.py --config C2 > $o/final_bench_c2.json 2> $o/final_bench_c2.err; echo "exit $?" >> $o/final_bench_c2.err
timeout 900 python bench.py --config C3 > $o/final_bench_c3.json 2> $o/final_bench_c3.err; echo "exit $?" >> $o/final_bench_c3.err
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $o/final_bench_ref.json 2> $o/final_bench_ref.err; echo "exit $?" >> $o/final_bench_ref.err
timeout 1200 /usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv \
  --log-file $o/final_launches.csv python bench.py --quick --steps 2 --warmup 1 --parity-edges 0 > $o/final_ncu_launch.log 2>&1; echo "exit $?" >> $o/final_ncu_launch.log
NB=2 QUERIES=prism6 timeout 1500 /usr/local/cuda/bin/ncu --set full --import-source on --clock-control none --kernel-name-base function \
  -k regex:"^(k_extend|k_walks)$" --launch-skip 2 --launch-count 2 -f -o $o/ncu_c4_prism6_final \
  python scripts/c4_ncu.py > $o/final_ncu_full.log 2>&1; echo "exit $?" >> $o/final_ncu_full.log
out=$o/final_ab_merge2.txt; : > $out
for v in def merge2 def merge2; do
  mg=""; [ $v == merge2 ] && mg=1
  env ${mg:+GCSM_MERGE2=1} timeout 900 python bench.py --quick --steps 8 --warmup 3 --parity-edges 0 2>>$o/final_ab_merge2.err | tail -1 | \
    python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$v', round(d['value']), round(d['ms_per_step'],2), {q: (round(x['ms_extend'],2), round(x['ms_walks'],2)) for q,x in d['per_query'].items()})" >> $out
done
