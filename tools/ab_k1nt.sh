#!/bin/bash
# K1 block-size A/B (FFSVA_K1_NT) on M1/M2/M3/M5 + parity of the default choice, on one B200.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/ab
python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_sdd_variants.py -q -x > gpurun_out/pytest_k1nt.log 2>&1
echo "parity rc=$?"; tail -3 gpurun_out/pytest_k1nt.log
for nt in ${NTS:-auto 256}; do
  for cfg in ${CONFIGS:-m1 m2 m3 m5}; do
    if [ "$nt" = auto ]; then unset FFSVA_K1_NT; else export FFSVA_K1_NT=$nt; fi
    timeout 600 python bench.py --config $cfg --steps ${STEPS:-1000} --warmup 5 --no-e2e --no-cpu-baseline \
      --online "" --online-tyolo "" > gpurun_out/ab/nt${nt}_${cfg}.json 2> gpurun_out/ab/nt${nt}_${cfg}.err
    python -c "import json;d=json.load(open('gpurun_out/ab/nt${nt}_${cfg}.json'));r=d['roofline'];print('nt$nt', '$cfg', round(d['value']), round(r['achieved']), round(r['frac'],3), {k:round(v,4) for k,v in r['kernel_ms'].items()})" || tail -3 gpurun_out/ab/nt${nt}_${cfg}.err
  done
done
unset FFSVA_K1_NT
