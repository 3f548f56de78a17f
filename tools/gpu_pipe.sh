#!/bin/bash
# Online runtime check on one B200: scheduler + parity GPU tests, then the default bench (M2 + paced online ladder)
# and the T-YOLO stage bench (new resize kernel).
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -30 gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_gpu.log
timeout 1500 python bench.py --steps 1000 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
python3 - <<'PY'
import json
d = json.load(open("gpurun_out/bench.json"))
print(d["value"], d["roofline"]["frac"], d["e2e"]["value"])
for r in d["online"]["runs"]:
    print(r["streams"], r.get("stages", ""), r["sustained"], round(r["latency_p99_s"], 3), r["backlog_frames_at_end"], r["mean_ms_per_tick"])
PY
timeout 900 python bench.py --config tyolo --steps 200 --warmup 5 > gpurun_out/bench_tyolo.json 2> gpurun_out/bench_tyolo.err; echo "tyolo rc=$?"
python3 -c "import json; d=json.load(open('gpurun_out/bench_tyolo.json')); print(d['value'], d['roofline']['frac'], d['roofline']['layer_ms'])"
