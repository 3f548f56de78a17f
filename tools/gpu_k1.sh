#!/bin/bash
# K1 check: parity tests + bench lines for M1 / M2 / M3 / M5.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/ab
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/pytest_parity.log 2>&1; echo "parity rc=$?"; tail -2 gpurun_out/pytest_parity.log
for cfg in ${CFGS:-m1 m2 m3 m5}; do
  timeout 600 python bench.py --config $cfg --steps ${STEPS:-300} --warmup 5 --online "" --no-e2e --no-cpu-baseline > gpurun_out/ab/k1_$cfg.json 2> gpurun_out/ab/k1_$cfg.err
  python3 -c "
import json; d=json.load(open('gpurun_out/ab/k1_$cfg.json')); r=d['roofline']
print('$cfg', round(d['value']), 'frac', round(r['frac'],3), 'K1ms', round(r['kernel_ms']['K1_sdd'],4), 'step', round(d['ms_per_step'],4), r['peak_source'])" || tail -3 gpurun_out/ab/k1_$cfg.err
done
