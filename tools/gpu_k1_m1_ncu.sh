#!/bin/bash
# ncu --set full capture of K1 (warp-segment kernel) at M1 (360p)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sdd -s 20 -c 1 -o gpurun_out/prof_k1_m1 -f \
  python bench.py --config m1 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --online "" > gpurun_out/ncu_k1_m1.log 2>&1
echo "ncu rc=$?"
python tools/ncu_brief.py gpurun_out/prof_k1_m1.ncu-rep 2>&1 | head -24
