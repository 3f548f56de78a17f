#!/bin/bash
# after the K1 shared-memory-limit fix: parity (incl. the fresh-process regression test), SNM + M2 bench lines,
# the K4 ncu capture, racecheck of the SDD -> SNM cascade.
cd "$(dirname "$0")/.."
python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x > gpurun_out/pytest_fix.log 2>&1; echo "parity rc=$?"; tail -2 gpurun_out/pytest_fix.log
timeout 900 python bench.py --config snm --steps 200 --warmup 5 --online "" --online-tyolo "" > gpurun_out/bench_snm.json 2> gpurun_out/bench_snm.err; echo "bench snm rc=$?"
timeout 900 python bench.py --config m2 --steps 1000 --warmup 5 --no-e2e --no-cpu-baseline --online "" --online-tyolo "" > gpurun_out/bench_m2_fix.json 2> gpurun_out/bench_m2_fix.err; echo "bench m2 rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:snm_kernel -s 10 -c 1 -o gpurun_out/prof_k4_snm -f \
  python bench.py --config snm --steps 20 --warmup 3 --no-e2e --no-cpu-baseline --online "" --online-tyolo "" > gpurun_out/ncu_full_k4.log 2>&1
echo "ncu full k4 rc=$?"
timeout 1500 compute-sanitizer --tool racecheck --error-exitcode 9 python tools/sanitize_run.py --no-tyolo > gpurun_out/sanitize_racecheck.log 2>&1
echo "sanitize racecheck rc=$?"; tail -2 gpurun_out/sanitize_racecheck.log
