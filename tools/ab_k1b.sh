#!/bin/bash
# K1 A/B (R row staged in shared memory; 128-thread CTAs at 16/SM) + parity of the new default, on one B200.
#   bash tools/ab_k1b.sh base old=FFSVA_K1_REFPRE=0,FFSVA_K1_MINB128=12 ...
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/ab
python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x > gpurun_out/pytest_k1ab.log 2>&1
echo "parity rc=$?"; tail -3 gpurun_out/pytest_k1ab.log
for spec in "$@"; do
  name=${spec%%=*}; defs=${spec#*=}
  if [ "$name" = "base" ]; then lib=$PWD/paper_conf_icpp_zhangcjzly18_b200/lib/libffsva.so; else
    lib=$(python -c "import __graft_entry__ as g; print(g.build_variant('$name', '$defs'.split(',') if '$defs' else []))"); fi
  for cfg in ${CONFIGS:-m1 m2 m3}; do
    FFSVA_LIB=$lib timeout 600 python bench.py --config $cfg --steps ${STEPS:-1000} --warmup 5 --no-e2e --no-cpu-baseline \
      --online "" --online-tyolo "" > gpurun_out/ab/${name}_${cfg}.json 2> gpurun_out/ab/${name}_${cfg}.err
    python -c "import json;d=json.load(open('gpurun_out/ab/${name}_${cfg}.json'));r=d['roofline'];print('$name', '$cfg', round(d['value']), round(r['achieved']), round(r['frac'],3), {k:round(v,4) for k,v in r['kernel_ms'].items()})" || tail -3 gpurun_out/ab/${name}_${cfg}.err
  done
done
