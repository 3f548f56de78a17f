#!/bin/bash
# ncu --set full capture of K4 (snm_kernel) on the SNM microbenchmark, plus the reforward GPU tests.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 600 python -m pytest tests/test_gpu_reforward.py -q > gpurun_out/pytest_reforward.log 2>&1; echo "reforward rc=$?"; tail -2 gpurun_out/pytest_reforward.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:snm_kernel -s 10 -c 1 -o gpurun_out/prof_k4_snm -f \
  python bench.py --config snm --steps 20 --warmup 3 --no-e2e --no-cpu-baseline --online "" > gpurun_out/ncu_full_k4.log 2>&1
echo "ncu k4 rc=$?"
python tools/ncu_summary.py gpurun_out/prof_k4_snm.ncu-rep > gpurun_out/ncu_full_k4_snm.json 2>&1; head -c 2500 gpurun_out/ncu_full_k4_snm.json
