#!/bin/bash
# Online runtime: scheduler GPU tests + the default bench (M2 + paced ladder + T-YOLO cascade).
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
timeout 900 python -m pytest tests/test_gpu_sched.py tests/test_gpu_reforward.py -q > gpurun_out/pytest_sched.log 2>&1; echo "sched rc=$?"; tail -2 gpurun_out/pytest_sched.log
timeout 1500 python bench.py --steps 1000 ${EXTRA} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
python3 - <<'PY'
import json
d = json.load(open("gpurun_out/bench.json"))
print(d["value"], d["roofline"]["frac"], d["e2e"]["value"])
for r in d["online"]["runs"]:
    print(r["streams"], r.get("stages", ""), r["sustained"], round(r["latency_p99_s"], 3), r["ticks"], r["backlog_frames_at_end"], {k: round(v, 2) for k, v in r["mean_ms_per_tick"].items()})
PY
