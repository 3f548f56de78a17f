#!/bin/bash
# 360p K1: band-of-two CTAs (default for rows of <= 128 chunks) vs CTA pairs (FFSVA_K1_NT=128); parity first.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/ab
python __graft_entry__.py > gpurun_out/build.log 2>&1 || exit 1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sdd_variants.py tests/test_gpu_sched.py -q -x > gpurun_out/pytest_band2.log 2>&1
echo "parity rc=$?"; tail -2 gpurun_out/pytest_band2.log
for nt in auto 128; do
  for cfg in m1 snm; do
    if [ $nt = auto ]; then unset FFSVA_K1_NT; else export FFSVA_K1_NT=$nt; fi
    timeout 600 python bench.py --config $cfg --steps 300 --warmup 5 --no-e2e --no-cpu-baseline --online "" --online-tyolo "" > gpurun_out/ab/b2_${nt}_${cfg}.json 2> gpurun_out/ab/b2_${nt}_${cfg}.err
    python -c "import json;d=json.load(open('gpurun_out/ab/b2_${nt}_${cfg}.json'));r=d['roofline'];print('$nt', '$cfg', round(d['value']), round(r['frac'],3), r['kernel_ms'])" || tail -2 gpurun_out/ab/b2_${nt}_${cfg}.err
  done
done
unset FFSVA_K1_NT
timeout 600 ncu --set full --clock-control none -k regex:sdd -s 20 -c 1 -o gpurun_out/prof_k1_m1_band2 -f python bench.py --config m1 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --online "" --online-tyolo "" > /dev/null 2>&1; echo "ncu rc=$?"
