#!/bin/bash
# ncu --set full capture of one K1 launch inside the paced online runtime (S streams of M2 content), to compare with
# the offline M2 capture (per-frame bytes, stalls)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
S=${S:-50000}
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:sdd_bulk -s ${SKIP:-260} -c 1 -o gpurun_out/prof_k1_online -f \
  python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --online "$S" --online-seconds 3 --online-tyolo "" \
  --online-tor "" > gpurun_out/ncu_online_full.log 2>&1
echo "ncu rc=$?"
python tools/ncu_brief.py gpurun_out/prof_k1_online.ncu-rep 2>&1 | head -24
