#!/bin/bash
# K4 ablation (A/B builds with parts compiled out; results wrong, timing only): which stage bounds the pipeline.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
for v in ${ABL:-0 1 2 4 6 7 8 15}; do
  python -c "import __graft_entry__ as g; g.build_variant('abl$v', ['FFSVA_K4_ABL=$v'])" > /dev/null 2>&1 || { echo "variant $v build failed"; continue; }
  FFSVA_LIB=paper_conf_icpp_zhangcjzly18_b200/lib/libffsva_abl$v.so timeout 300 python bench.py --config snm --steps 30 --warmup 3 \
    --online "" --no-e2e --no-cpu-baseline > gpurun_out/abl$v.json 2> gpurun_out/abl$v.err
  python3 -c "import json; d=json.load(open('gpurun_out/abl$v.json')); print('abl $v', round(d['roofline']['kernel_ms']['K4_snm'], 4), 'ms')" 2>&1 | tail -1
done
