#!/bin/bash
# Build + full GPU test suite + T-YOLO stage bench on one B200.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -30 gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -8 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --config tyolo --steps 200 --warmup 5 > gpurun_out/bench_tyolo.json 2> gpurun_out/bench_tyolo.err; echo "tyolo rc=$?"
python3 -c "import json; d=json.load(open('gpurun_out/bench_tyolo.json')); print(d['value'], d['roofline']['frac'], d['roofline']['layer_ms'])"
