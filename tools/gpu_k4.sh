#!/bin/bash
# Build + full GPU tests + SNM / T-YOLO / M2 benches on one B200.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; tail -30 gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -8 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --config snm --steps 100 --warmup 5 --online "" --no-e2e > gpurun_out/bench_snm.json 2> gpurun_out/bench_snm.err; echo "snm rc=$?"
python3 -c "import json; d=json.load(open('gpurun_out/bench_snm.json')); r=d['snm_roofline']; print('snm', r['survivors_per_s'], r['frac'], d['roofline']['kernel_ms'])"
timeout 900 python bench.py --config tyolo --steps 200 --warmup 5 > gpurun_out/bench_tyolo.json 2> gpurun_out/bench_tyolo.err; echo "tyolo rc=$?"
python3 -c "import json; d=json.load(open('gpurun_out/bench_tyolo.json')); print(d['value'], d['roofline']['frac'], d['roofline']['layer_ms'])"
timeout 1500 python bench.py --steps 1000 > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
python3 - <<'PY'
import json
d = json.load(open("gpurun_out/bench.json"))
print(d["value"], d["roofline"]["frac"], d["e2e"]["value"], d["snm_roofline"])
for r in d["online"]["runs"]:
    print(r["streams"], r.get("stages", ""), r["sustained"], round(r["latency_p99_s"], 3), r["ticks"], r["backlog_frames_at_end"], r["mean_ms_per_tick"])
PY
