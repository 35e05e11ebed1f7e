#!/bin/bash
# round 2: A/B of the current kernel vs round 1 on every config + the parity suite
cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
: > gpurun_out/ab2.txt
for c in ${CONFIGS:-gh_work dblp bx yg_work bx_work}; do
  for v in r1base cur; do
    if [ $v = cur ]; then L=""; else L=build_variants/libgmbe_$v.so; fi
    echo "== $c $v" >> gpurun_out/ab2.txt
    GMBE_LIB=$L timeout 300 python scripts/sweep.py $c "" "" ${SWEEP_EXTRA} >> gpurun_out/ab2.txt 2>&1
  done
done
cat gpurun_out/ab2.txt
timeout 1500 python -m pytest tests -m gpu -x -q --deselect tests/test_sanitizer.py ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -15 gpurun_out/pytest_gpu.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_dblp2.csv python bench.py --config dblp --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/bench_dblp_ncu2.log 2>&1
python scripts/launch_summary.py gpurun_out/launches_dblp2.csv | head -14
GMBE_SANITIZER_LOG_DIR=gpurun_out timeout 1800 python -m pytest tests/test_sanitizer.py -x -q -k "racecheck or synccheck" > gpurun_out/pytest_sanitizer.log 2>&1; echo "sanitizer rc=$?" >> gpurun_out/pytest_sanitizer.log
tail -3 gpurun_out/pytest_sanitizer.log; grep -h "SUMMARY" gpurun_out/r02_sanitizer_*.log
