#!/bin/bash
# Online runtime: scheduler / re-forwarding GPU tests, then paced runs at fixed stream counts (SDD + SNM, M2 content).
#   COUNTS="55000,58000"  SECONDS_=10
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x -k "sched or reforward or online" > gpurun_out/pytest_sched.log 2>&1; echo "pytest rc=$?"
tail -3 gpurun_out/pytest_sched.log
timeout 1500 python bench.py --steps 50 --warmup 5 --no-e2e --no-cpu-baseline --online "${COUNTS:-55000,58000,61000}" \
  --online-seconds ${SECONDS_:-10} --online-tyolo "" --online-tor "" > gpurun_out/online_ab.json 2> gpurun_out/online_ab.err
echo "bench rc=$?"
python3 - <<'PY'
import json
d = json.load(open("gpurun_out/online_ab.json"))
print("offline", round(d["value"]), "streams by throughput", d["sustained_streams_30fps"])
for r in d["online"]["runs"]:
    print(r["streams"], r["sustained"], round(r["latency_p99_s"], 3), r["ticks"], round(r["decided_fps"]), r["backlog_slope_per_stream"],
          {k: round(v, 2) for k, v in r["mean_ms_per_tick"].items()})
PY
