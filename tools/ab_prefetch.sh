#!/bin/bash
# K1 L2-prefetch A/B (FFSVA_K1_PREFETCH = frames ahead) on M2 / M3 / M5, plus parity with the prefetch on.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/ab
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
FFSVA_K1_PREFETCH=9 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/pytest_parity.log 2>&1; echo "parity rc=$?"; tail -2 gpurun_out/pytest_parity.log
for cfg in m2 m3 m5; do for d in 0 3 6 9 12 18; do
  FFSVA_K1_PREFETCH=$d timeout 600 python bench.py --config $cfg --steps 300 --warmup 5 --online "" --no-e2e --no-cpu-baseline > gpurun_out/ab/pf_${cfg}_$d.json 2> gpurun_out/ab/pf_${cfg}_$d.err
  python3 -c "
import json; d=json.load(open('gpurun_out/ab/pf_${cfg}_$d.json')); r=d['roofline']
print('$cfg d=$d', round(d['value']), 'frac', round(r['frac'],3), 'K1ms', round(r['kernel_ms']['K1_sdd'],4))" || tail -3 gpurun_out/ab/pf_${cfg}_$d.err
done; done
