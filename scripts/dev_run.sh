timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -p no:cacheprovider > gpurun_out/gpu_tests.txt 2>&1; tail -3 gpurun_out/gpu_tests.txt
GCSM_TRACE=1 timeout 300 python bench.py --quick --serial --steps 3 --warmup 2 --queries c4 > gpurun_out/tr.json 2> gpurun_out/tr.err; grep "gcsm kern" gpurun_out/tr.err | tail -2
VARIANTS="old new" bash scripts/ab.sh
