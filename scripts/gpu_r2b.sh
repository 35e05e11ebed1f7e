#!/bin/bash
# round 2, second GPU pass: suite (incl. schedulers), sanitizers, timings, phases, dblp launch list
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q --deselect tests/test_sanitizer.py > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
: > gpurun_out/times.txt
for c in gh_work dblp bx yg_work bx_work gh; do
  echo "== $c" >> gpurun_out/times.txt
  timeout 600 python scripts/sweep.py $c "" "" "scheduler=warp" "scheduler=block" "debug=1024" >> gpurun_out/times.txt 2>&1
done
GMBE_LIB=paper_conf_sc_panhlzwc23_b200/libgmbe_prof.so timeout 600 python scripts/phase_run.py gh_work dblp bx bx_work > gpurun_out/phases.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_dblp.csv python bench.py --config dblp --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/bench_dblp_ncu.log 2>&1
GMBE_SANITIZER_LOG_DIR=gpurun_out timeout 2400 python -m pytest tests/test_sanitizer.py -x -q > gpurun_out/pytest_sanitizer.log 2>&1; echo "sanitizer rc=$?" >> gpurun_out/pytest_sanitizer.log
tail -5 gpurun_out/pytest_gpu.log; cat gpurun_out/times.txt gpurun_out/phases.txt; tail -5 gpurun_out/pytest_sanitizer.log
