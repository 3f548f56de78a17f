#!/bin/bash
# K1 at 360p: CTA-pair bulk kernel vs the band (register-streaming) kernel
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/ab
python __graft_entry__.py > gpurun_out/build.log 2>&1 || exit 1
for k in pair stream; do
  for cfg in m1 m2; do
    if [ $k = stream ]; then export FFSVA_SDD_KERNEL=stream; else unset FFSVA_SDD_KERNEL; fi
    timeout 600 python bench.py --config $cfg --steps 500 --warmup 5 --no-e2e --no-cpu-baseline --online "" --online-tyolo "" > gpurun_out/ab/k_${k}_${cfg}.json 2> gpurun_out/ab/k_${k}_${cfg}.err
    python -c "import json;d=json.load(open('gpurun_out/ab/k_${k}_${cfg}.json'));r=d['roofline'];print('$k', '$cfg', round(d['value']), round(r['frac'],3), r['kernel_ms'])" || tail -2 gpurun_out/ab/k_${k}_${cfg}.err
  done
done
