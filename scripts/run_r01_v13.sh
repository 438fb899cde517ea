set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_r01_v13.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_r01_v13.txt 2>&1
bash scripts/evidence3.sh r01_v13
