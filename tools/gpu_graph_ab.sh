#!/bin/bash
# Online runtime with and without per-stage CUDA graphs (FFSVA_SCHED_GRAPH), GPU scheduler tests, sanitizers.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/graph_ab
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 900 python -m pytest tests/test_gpu_sched.py tests/test_gpu_reforward.py -q -rf > gpurun_out/graph_ab/pytest.log 2>&1
echo "pytest rc=$?"; tail -3 gpurun_out/graph_ab/pytest.log
for g in 1 0; do
  FFSVA_SCHED_GRAPH=$g timeout 900 python bench.py --steps 20 --warmup 5 --no-e2e --no-cpu-baseline --online=auto \
    --online-tyolo= --online-tor= --online-confirm-seconds 10 > gpurun_out/graph_ab/online_g$g.json 2> gpurun_out/graph_ab/online_g$g.err
  echo "graph=$g rc=$?"; python tools/show_online.py gpurun_out/graph_ab/online_g$g.json | head -12
done
if [ -n "$SANITIZE" ]; then bash tools/gpu_sanitize.sh; fi
