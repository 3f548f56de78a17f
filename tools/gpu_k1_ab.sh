#!/bin/bash
# A/B of the narrow-row K1 configurations (warp-segment groups x stages) on M1 against the one-CTA-per-band kernel.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/k1ab
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -30 gpurun_out/build.log; exit 1; }
if [ -n "$TESTS" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -rf -k "$TESTS" > gpurun_out/k1ab/pytest.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/k1ab/pytest.log
fi
for rep in 1 2; do
for v in ${VARIANTS:-seg2,5 seg2,4 seg3,8 seg1,6 pipe2,2 old}; do
  unset FFSVA_K1_NT FFSVA_K1_PIPE FFSVA_K1_SEG FFSVA_K1_GRP
  case $v in
    grp*) export FFSVA_K1_GRP=${v#grp} ;;
    old) export FFSVA_K1_NT=1282 ;;
    pipe*) export FFSVA_K1_NT=1283 FFSVA_K1_PIPE=${v#pipe} ;;
    seg*) export FFSVA_K1_NT=1284 FFSVA_K1_SEG=${v#seg} ;;
  esac
  for cfg in ${CONFIGS:-m1}; do
  timeout 600 python bench.py --config $cfg --steps 300 --warmup 5 --online= --no-e2e --no-cpu-baseline > gpurun_out/k1ab/${cfg}_$v.json 2> gpurun_out/k1ab/${cfg}_$v.err
  python -c "import json;d=json.load(open('gpurun_out/k1ab/${cfg}_$v.json'));r=d['roofline'];print('$cfg $v', round(d['value']), 'step', round(d['ms_per_step'],4), 'frac', round(r.get('frac'),3), {k:round(x,4) for k,x in r.get('kernel_ms').items()})" || tail -3 gpurun_out/k1ab/${cfg}_$v.err
  done
done
done
unset FFSVA_K1_NT FFSVA_K1_PIPE FFSVA_K1_SEG FFSVA_K1_GRP
if [ -n "$NCU" ]; then
  FFSVA_K1_GRP=$NCU timeout 600 ncu --set full --clock-control none --import-source on -k regex:sdd_grp -s 10 -c 1 -o gpurun_out/k1ab/prof_m1 -f \
    python bench.py --config m1 --steps 20 --warmup 3 --online= --no-e2e --no-cpu-baseline > gpurun_out/k1ab/ncu.log 2>&1; echo "ncu rc=$?"
fi
