#!/bin/bash
# K4 iteration: SNM parity tests (short timeout: a pipeline deadlock must not hold the box), then the standalone
# SNM bench.   K=expr selects tests (default: snm-related)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -30 gpurun_out/build.log; exit 1; }
timeout 300 python -m pytest tests -m gpu -x -q -k "${K:-snm or smoke or fullsize}" > gpurun_out/pytest_k4.log 2>&1; echo "pytest rc=$?"
tail -15 gpurun_out/pytest_k4.log
timeout 300 python bench.py --config snm --steps 50 --warmup 5 --online "" --no-e2e --no-cpu-baseline > gpurun_out/bench_snm.json 2> gpurun_out/bench_snm.err; echo "snm rc=$?"
tail -3 gpurun_out/bench_snm.err
python3 -c "import json; d=json.load(open('gpurun_out/bench_snm.json')); r=d['snm_roofline']; print('snm', r['survivors_per_s'], r['frac'], d['roofline']['kernel_ms'])"
