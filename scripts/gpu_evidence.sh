#!/bin/bash
# round 2 evidence: bench lines (all shapes), reference arm, launch list, ncu full of k_enum, Fig 9
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm --format=csv > gpurun_out/ev_clocks.txt
[ -x scripts/l2peak ] || nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o scripts/l2peak scripts/l2peak.cu
./scripts/l2peak > gpurun_out/ev_l2peak.txt 2>&1
timeout 900 python bench.py > gpurun_out/ev_bench_gh_work.json 2> gpurun_out/ev_bench_gh_work.err
for c in dblp bx bx_work yg_work gh yg; do
  timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/ev_bench_$c.json 2> gpurun_out/ev_bench_$c.err
done
timeout 900 python bench.py --impl reference > gpurun_out/ev_bench_ref_gh_work.json 2> gpurun_out/ev_bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev_launches_gh_work.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ev_bench_under_ncu.log 2>&1
python scripts/launch_summary.py gpurun_out/ev_launches_gh_work.csv > gpurun_out/ev_launches_gh_work.txt 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_enum$" -s 1 -c 1 -o gpurun_out/ev_gh_work python scripts/ncu_target.py gh_work > gpurun_out/ev_ncu.log 2>&1
python scripts/ncu_summary.py gpurun_out/ev_gh_work.ncu-rep --json gpurun_out/ev_ncu_gh_work.json > gpurun_out/ev_ncu_gh_work.txt 2>&1
for c in gh_work bx_work; do timeout 900 python scripts/fig9_sched.py $c --out gpurun_out/ev_fig9_$c.json > gpurun_out/ev_fig9_$c.log 2>&1; done
for f in gpurun_out/ev_bench_*.json; do echo "== $f"; cat $f | cut -c1-400; done
cat gpurun_out/ev_launches_gh_work.txt | head -12; cat gpurun_out/ev_ncu_gh_work.txt | head -24; tail -2 gpurun_out/ev_fig9_*.log
for c in gh_work bx_work dblp; do timeout 900 python scripts/shard_times.py $c 2 4 8 mode=cost > gpurun_out/ev_shards_$c.json 2>&1; done
cat gpurun_out/ev_shards_*.json | cut -c1-600
