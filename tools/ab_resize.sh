#!/bin/bash
# T-YOLO resize A/B: output rows per CTA (FFSVA_TYOLO_RESIZE_ROWS), per-layer profile of 256 720p frames.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/ab
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
for R in 1 2 3 4 6 9 12; do
  FFSVA_TYOLO_RESIZE_ROWS=$R timeout 300 python tools/tyolo_profile.py --frames 256 --iters 10 --out gpurun_out/ab/resize_$R.json > gpurun_out/ab/resize_$R.log 2>&1
  grep -E '^resize' gpurun_out/ab/resize_$R.log | sed "s/^/R=$R /" || tail -3 gpurun_out/ab/resize_$R.log
done
