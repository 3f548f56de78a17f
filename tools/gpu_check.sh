#!/bin/bash
# One gpurun call: build, GPU tests, smoke, bench, ncu launch list + full captures of K1 and K4.
#   BENCH="--steps 2000 --warmup 10"  run bench.py with these args
#   NCU=1                              ncu launch list + --set full captures (profiles come back in gpurun_out/)
#   PYTEST_K="expr"                    subset of GPU tests (pytest -k)
#   SKIP_TESTS=1                       skip pytest + smoke
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
nvidia-smi > gpurun_out/nvidia-smi.txt 2>&1
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -30 gpurun_out/build.log; exit 1; }
if [ -z "$SKIP_TESTS" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
  tail -25 gpurun_out/pytest_gpu.log
  timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/smoke.log
fi
if [ -n "$BENCH" ]; then
  timeout 900 python bench.py $BENCH > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
  cat gpurun_out/bench.json; tail -5 gpurun_out/bench.err
fi
if [ -n "$NCU" ]; then
  CFG=${NCU_CONFIG:-m2}
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"sdd|compact|snm" -s 60 -c 60 --csv \
    --log-file gpurun_out/launches_${CFG}.csv \
    python bench.py --config $CFG --steps 40 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_list.log 2>&1
  echo "ncu list rc=$?"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:sdd -s 40 -c 2 -o gpurun_out/prof_k1_${CFG} -f \
    python bench.py --config $CFG --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_k1.log 2>&1
  echo "ncu full k1 rc=$?"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:snm_kernel -s 20 -c 2 -o gpurun_out/prof_k4_${CFG} -f \
    python bench.py --config $CFG --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_k4.log 2>&1
  echo "ncu full k4 rc=$?"
fi
