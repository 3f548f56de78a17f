#!/bin/bash
# K4 wait-time profile (A/B build with FFSVA_K4_PROF: CTA 0 prints its per-wait clock totals per launch)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
python -c "import __graft_entry__ as g; g.build_variant('prof', ['FFSVA_K4_PROF=1'] + '${EXTRA}'.split())" > gpurun_out/build_prof.log 2>&1 || { echo "prof build failed"; tail gpurun_out/build_prof.log; exit 1; }
FFSVA_LIB=paper_conf_icpp_zhangcjzly18_b200/lib/libffsva_prof.so timeout 300 python bench.py --config snm --steps 10 --warmup 3 \
    --online "" --no-e2e --no-cpu-baseline > gpurun_out/k4prof.out 2> gpurun_out/k4prof.err
grep K4PROF gpurun_out/k4prof.out | tail -3
