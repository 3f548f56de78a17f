#!/bin/bash
# ncu --set full captures of the T-YOLO conv kernel: launch k of a 256-frame profile run (k = 1: L1, 2: L2, 8: L8).
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
python __graft_entry__.py > gpurun_out/build.log 2>&1
for L in ${LAYERS:-1 2 8}; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:tyolo_conv -s $((L - 1)) -c 1 \
    -o gpurun_out/prof_tyolo_L$L -f python tools/tyolo_profile.py --frames 256 --iters 1 > gpurun_out/ncu_tyolo_L$L.log 2>&1
  echo "L$L rc=$?"
done
