#!/bin/bash
# the driver's default bench line (M2, e2e, CPU baseline, online ladders) + an ncu capture of K1 at M1
cd "$(dirname "$0")/.."
python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
nproc > gpurun_out/nproc.txt; python -c "import os; print(len(os.sched_getaffinity(0)))" >> gpurun_out/nproc.txt
timeout 1800 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sdd -s 20 -c 1 -o gpurun_out/prof_k1_m1 -f \
  python bench.py --config m1 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --online "" --online-tyolo "" > gpurun_out/ncu_k1_m1.log 2>&1
echo "ncu m1 rc=$?"
