#!/bin/bash
# bench step overlap A/B: --streams 1/2/3 on M2, M3, M4 (10 %), M1.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/ab
python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
for ns in ${NS:-1 2 3}; do
  for cfg in ${CONFIGS:-m2 m3 m4_10 m1}; do
    timeout 600 python bench.py --config $cfg --streams $ns --steps ${STEPS:-1000} --warmup 5 --no-e2e --no-cpu-baseline \
      --online "" --online-tyolo "" > gpurun_out/ab/str${ns}_${cfg}.json 2> gpurun_out/ab/str${ns}_${cfg}.err
    python -c "import json;d=json.load(open('gpurun_out/ab/str${ns}_${cfg}.json'));r=d['roofline'];print('streams$ns', '$cfg', round(d['value']), round(d['ms_per_step'],4), round(r['frac'],3), d['gpu_launches'])" || tail -3 gpurun_out/ab/str${ns}_${cfg}.err
  done
done
