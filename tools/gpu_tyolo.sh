#!/bin/bash
# T-YOLO check: GPU tests of the stage (and the online cascade), then the stage bench.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_tyolo.py tests/test_gpu_sched.py -q -x > gpurun_out/pytest_tyolo.log 2>&1; echo "tyolo tests rc=$?"; tail -4 gpurun_out/pytest_tyolo.log
timeout 900 python bench.py --config tyolo --steps 200 --warmup 5 > gpurun_out/bench_tyolo.json 2> gpurun_out/bench_tyolo.err; echo "tyolo rc=$?"
python3 -c "import json; d=json.load(open('gpurun_out/bench_tyolo.json')); print(d['value'], d['roofline']['frac'], d['roofline']['layer_ms'])" || tail -5 gpurun_out/bench_tyolo.err
