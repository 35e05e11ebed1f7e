#!/bin/bash
# Tail analysis + the N>1 bench code path on one GPU (GMBE_BENCH_SHARE_GPU=1: 2 ranks on GPU 0, gloo)
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
timeout 250 python scripts/root_phases.py gh_work 6 > gpurun_out/rp2_gh_work.txt 2>&1
timeout 250 python scripts/root_phases.py bx 6 > gpurun_out/rp2_bx.txt 2>&1
timeout 250 python scripts/root_alone.py gh_work 56504 56496 56488 > gpurun_out/ra_gh_work.txt 2>&1
timeout 250 python scripts/root_alone.py bx 105072 104952 105112 > gpurun_out/ra_bx.txt 2>&1
for p in dynamic interleave cost; do
GMBE_BENCH_SHARE_GPU=1 timeout 400 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
   bench.py --gpus 2 --steps 5 --warmup 3 --partition $p > gpurun_out/bench_share2_$p.json 2> gpurun_out/bench_share2_$p.err
done
cat gpurun_out/rp2_*.txt gpurun_out/ra_*.txt gpurun_out/bench_share2_*.json; tail -5 gpurun_out/bench_share2_dynamic.err
