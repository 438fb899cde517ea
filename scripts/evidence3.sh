#!/bin/bash
# Round evidence (r01 v11): full bench line (C2 default), ncu launch list, full capture of the top kernel (c4's
# k_last4) and of the GPU estimator's kernels, C3/C4 bench lines, torchrun N=2 plumbing (emulated on one GPU),
# the reference arm, smoke(). Usage (under gpurun): bash scripts/evidence3.sh <tag>
T=${1:-dev}
timeout 900 python bench.py > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$T.csv \
    python bench.py --steps 2 --warmup 1 --quick --serial > gpurun_out/ncu_launch_$T.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_last4" -s 1 -c 1 -o gpurun_out/prof_c4_$T -f \
    python bench.py --steps 1 --warmup 1 --quick --serial --queries c4 > gpurun_out/ncu_c4_$T.txt 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_walks_l1|k_copy" -s 2 -c 2 -o gpurun_out/prof_est_$T -f \
    python bench.py --steps 1 --warmup 1 --quick --serial > gpurun_out/ncu_est_$T.txt 2>&1
timeout 900 python bench.py --config C3 > gpurun_out/bench_c3_$T.json 2> gpurun_out/bench_c3_$T.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29517 \
    bench.py --gpus 2 --emulate --quick --steps 2 --warmup 1 > gpurun_out/bench_emul2_$T.json 2> gpurun_out/bench_emul2_$T.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref_$T.json 2> gpurun_out/bench_ref_$T.err
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_$T.txt 2>&1
