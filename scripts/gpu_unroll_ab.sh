cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
VARIANTS="u1 u2 u4 u8" CONFIGS="gh_work bx dblp" SHARD_VARIANTS="u1 u4 u8" SHARD_CONFIG=gh_work bash scripts/gpu_variants.sh > /dev/null 2>&1
for v in u1 u4 u8; do GMBE_LIB=build_variants/libgmbe_$v.so timeout 300 python scripts/shard_times.py bx 8 | python -c "import sys,json; d=json.load(sys.stdin); print('$v bx shard8', d['n1_ms'], d['n8']['max_ms'], d['n8']['imbalance'])" >> gpurun_out/variants.txt 2>&1; done
GMBE_BENCH_SHARE_GPU=1 timeout 400 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --partition dynamic > gpurun_out/bench_share2_dynamic.json 2> gpurun_out/bench_share2_dynamic.err
cat gpurun_out/variants.txt gpurun_out/bench_share2_dynamic.json; grep -i error gpurun_out/bench_share2_dynamic.err | head -5
