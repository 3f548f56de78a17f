#!/bin/bash
# Build + GPU tests + bench lines for every §8(d) config (M1, M2, M3, M4 sweep, M5, SNM, T-YOLO) on one B200.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
nvidia-smi > gpurun_out/nvidia-smi.txt 2>&1
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -30 gpurun_out/build.log; exit 1; }
if [ -z "$NO_TESTS" ]; then
  timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
fi
for CFG in ${CFGS:-m1 m2 m3 m4_1 m4_10 m4_50 m5 snm}; do
  timeout 900 python bench.py --config $CFG --steps ${STEPS:-200} --warmup 5 --online "" ${EXTRA} > gpurun_out/bench_$CFG.json 2> gpurun_out/bench_$CFG.err
  echo "bench $CFG rc=$?"; cut -c1-400 gpurun_out/bench_$CFG.json
done
