#!/bin/bash
# K1 after the instruction trims: parity + M1/M2/M3 bench lines + an ncu --set full capture of K1 at M2.
cd "$(dirname "$0")/.."
NTS=auto CONFIGS="${CONFIGS:-m1 m2 m3}" bash tools/ab_k1nt.sh > gpurun_out/ab_k1d.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sdd -s 40 -c 1 -o gpurun_out/prof_k1_m2_${TAG:-d} -f \
    python bench.py --config m2 --steps 20 --warmup 3 --no-e2e --no-cpu-baseline --online "" --online-tyolo "" > gpurun_out/ncu_k1d.log 2>&1
echo "ncu rc=$?" >> gpurun_out/ab_k1d.log
