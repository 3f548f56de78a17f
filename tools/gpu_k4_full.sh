#!/bin/bash
# K4: all GPU tests, smoke, then an ncu --set full capture of snm_kernel on the SNM microbenchmark.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -30 gpurun_out/build.log; exit 1; }
if [ -z "$SKIP_TESTS" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -6 gpurun_out/pytest_gpu.log
  timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke.log
fi
timeout 300 python bench.py --config snm --steps 100 --warmup 5 --online "" --no-e2e --no-cpu-baseline > gpurun_out/bench_snm.json 2> gpurun_out/bench_snm.err; echo "snm rc=$?"
python3 -c "import json; d=json.load(open('gpurun_out/bench_snm.json')); r=d['snm_roofline']; print('snm', r['survivors_per_s'], r['frac'], d['roofline']['kernel_ms'], d.get('clocks'))"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:snm_kernel -s 10 -c 1 -o gpurun_out/prof_k4_snm -f \
  python bench.py --config snm --steps 20 --warmup 3 --no-e2e --no-cpu-baseline --online "" > gpurun_out/ncu_full_k4.log 2>&1
echo "ncu k4 rc=$?"
python tools/ncu_summary.py gpurun_out/prof_k4_snm.ncu-rep > gpurun_out/ncu_full_k4_snm.json 2>&1
python tools/ncu_brief.py gpurun_out/prof_k4_snm.ncu-rep 2>&1 | head -40
