#!/bin/bash
# New-feature GPU checks: f3/f2/f4 tests first (fast feedback), then the whole GPU suite, then the f4 study.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_sdd_variants.py tests/test_gpu_reforward.py tests/test_gpu_sched.py -q -x \
  > gpurun_out/pytest_new.log 2>&1; echo "new tests rc=$?"; tail -30 gpurun_out/pytest_new.log
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "gpu suite rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 900 python tools/batch_policy_study.py --seconds 1.0 > gpurun_out/batch_policy.log 2>&1; echo "study rc=$?"
tail -60 gpurun_out/batch_policy.log
