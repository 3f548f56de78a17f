#!/bin/bash
# K1 ring-kernel A/B on one B200: K1 parity tests, then bench lines per (config, variant, ring knobs).
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
for cfg in ${CFGS:-m2 m3 m1 m5}; do
  run ${cfg}_pair $cfg FFSVA_SDD_KERNEL=pair
  run ${cfg}_auto $cfg
  for c in ${CTAS:-1 2 3}; do for sl in ${SLOTS:-8192 16384 32768}; do
    run ${cfg}_ring_c${c}_s${sl} $cfg FFSVA_SDD_KERNEL=ring FFSVA_SDD_RING_CTAS=$c FFSVA_SDD_RING_SLOT=$sl
  done; done
done
