#!/bin/bash
# A/B of K1 build variants on the GPU: bench each (no e2e, no cpu baseline), print value + K1 GB/s.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
for spec in "$@"; do
  name=${spec%%=*}; defs=${spec#*=}
  if [ "$name" = "base" ]; then lib=$PWD/paper_conf_icpp_zhangcjzly18_b200/lib/libffsva.so; else
    lib=$(python -c "import __graft_entry__ as g; print(g.build_variant('$name', '$defs'.split(',') if '$defs' else []))"); fi
  for cfg in ${CONFIGS:-m2}; do
    FFSVA_LIB=$lib timeout 600 python bench.py --config $cfg --steps ${STEPS:-1000} --warmup 5 --no-e2e --no-cpu-baseline > gpurun_out/ab_${name}_${cfg}.json 2> gpurun_out/ab_${name}_${cfg}.err
    python -c "import json;d=json.load(open('gpurun_out/ab_${name}_${cfg}.json'));r=d['roofline'];print('$name', '$cfg', round(d['value']), round(r['achieved']), round(r['frac'],3), {k:round(v,4) for k,v in r['kernel_ms'].items()})" || tail -3 gpurun_out/ab_${name}_${cfg}.err
  done
done
