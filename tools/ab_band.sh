#!/bin/bash
# K1 band-kernel A/B on one B200: parity tests of K1, then bench lines per (config, variant, band smem target).
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/ab
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > gpurun_out/pytest_parity.log 2>&1; echo "parity rc=$?"; tail -3 gpurun_out/pytest_parity.log
run() {  # name config env...
  local name=$1 cfg=$2; shift 2
  env "$@" timeout 600 python bench.py --config $cfg --steps ${STEPS:-300} --warmup 5 --online "" --no-e2e --no-cpu-baseline \
    > gpurun_out/ab/$name.json 2> gpurun_out/ab/$name.err
  python3 -c "
import json; d=json.load(open('gpurun_out/ab/$name.json')); r=d['roofline']
print('$name', round(d['value']), 'frac', round(r['frac'],3), 'K1ms', round(r['kernel_ms']['K1_sdd'],4), 'step', round(d['ms_per_step'],4))" 2>/dev/null || { echo "$name FAILED"; tail -5 gpurun_out/ab/$name.err; }
}
for cfg in ${CFGS:-m1 m2 m3 snm}; do
  run ${cfg}_auto $cfg
  run ${cfg}_pair $cfg FFSVA_SDD_KERNEL=pair
  for t in ${TARGETS:-60000 100000 150000}; do run ${cfg}_band$t $cfg FFSVA_SDD_KERNEL=band FFSVA_SDD_BAND_SMEM=$t; done
done
