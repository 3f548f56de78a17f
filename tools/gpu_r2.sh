#!/bin/bash
# Round-2 GPU pass: build, all GPU tests (no -x: every failure reported), smoke, a short bench, and the N > 1 bench
# path on the one GPU (two ranks sharing cuda:0 over gloo).
#   PYTEST_K="expr"  subset;  BENCH="args"  bench.py args (default short m2);  SKIP_TESTS=1;  SKIP_DIST=1
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
nvidia-smi > gpurun_out/nvidia-smi.txt 2>&1
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -30 gpurun_out/build.log; exit 1; }
if [ -z "$SKIP_TESTS" ]; then
  timeout 2400 python -m pytest tests -m gpu -q -rf ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
  tail -30 gpurun_out/pytest_gpu.log
  timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/smoke.log
fi
B=${BENCH:---steps 40 --warmup 5 --online=}
timeout 900 python bench.py $B > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
cut -c1-1500 gpurun_out/bench.json; tail -5 gpurun_out/bench.err
if [ -z "$SKIP_DIST" ]; then
  timeout 900 python bench.py --gpus 2 --dist-backend gloo --steps 20 --warmup 3 --online= --no-cpu-baseline \
    > gpurun_out/bench_g2.json 2> gpurun_out/bench_g2.err; echo "bench g2 rc=$?"
  cut -c1-1500 gpurun_out/bench_g2.json; tail -5 gpurun_out/bench_g2.err
  timeout 900 python bench.py --gpus 2 --dist-backend gloo --config m5 --steps 10 --warmup 3 --no-cpu-baseline \
    --no-e2e > gpurun_out/bench_g2_m5.json 2> gpurun_out/bench_g2_m5.err; echo "bench g2 m5 rc=$?"
  cut -c1-1500 gpurun_out/bench_g2_m5.json; tail -5 gpurun_out/bench_g2_m5.err
fi
