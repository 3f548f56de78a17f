#!/bin/bash
# compute-sanitizer passes: racecheck to completion on the minimal K1 / K3 / K4 run, memcheck and synccheck on the
# full sanitize_run.py path set. Logs come back under gpurun_out/sanitize/.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/sanitize
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 2400 $CS --tool racecheck --racecheck-report hazard --print-limit 50 python tools/sanitize_run.py --minimal \
  > gpurun_out/sanitize/racecheck_minimal.log 2>&1; echo "racecheck rc=$?"; tail -4 gpurun_out/sanitize/racecheck_minimal.log
timeout 1500 $CS --tool memcheck --print-limit 50 python tools/sanitize_run.py > gpurun_out/sanitize/memcheck.log 2>&1
echo "memcheck rc=$?"; tail -3 gpurun_out/sanitize/memcheck.log
timeout 1500 $CS --tool synccheck --print-limit 50 python tools/sanitize_run.py > gpurun_out/sanitize/synccheck.log 2>&1
echo "synccheck rc=$?"; tail -3 gpurun_out/sanitize/synccheck.log
