#!/bin/bash
# Per-kernel device times inside the paced online runtime (M2 content, S streams): ncu launch list of K1 / K3 / K4
# over a few ticks (ncu serialises launches, so only the per-launch durations and their ratios are meaningful).
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 600 python __graft_entry__.py > gpurun_out/build.log 2>&1 || { echo BUILD FAILED; exit 1; }
S=${S:-50000}
timeout 900 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu-baseline --online "$S" --online-seconds 3 \
  --online-tyolo "" --online-tor "" > gpurun_out/online_$S.json 2> gpurun_out/online_$S.err
echo "online rc=$?"; python3 -c "
import json; d=json.load(open('gpurun_out/online_$S.json')); r=d['online']['runs'][0]
print({k: r[k] for k in ('streams','sustained','latency_p99_s','ticks','mean_ms_per_tick','decided_fps','offered_fps')})"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"sdd|compact|snm" -s 400 -c 60 --csv \
  --log-file gpurun_out/launches_online.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu-baseline \
  --online "$S" --online-seconds 3 --online-tyolo "" --online-tor "" > gpurun_out/ncu_online.log 2>&1
echo "ncu rc=$?"
python3 - <<'PY'
import csv, collections
rows = [r for r in csv.reader(open("gpurun_out/launches_online.csv")) if len(r) > 10]
h = rows[0]; ik = h.index("Kernel Name"); iv = h.index("Metric Value"); iu = h.index("Metric Unit")
agg = collections.defaultdict(list)
for r in rows[1:]:
    v = float(r[iv].replace(",", "")); v = v / 1000 if r[iu] == "nsecond" else (v * 1000 if r[iu] == "msecond" else v)
    agg[r[ik].split("(")[0][-40:]].append(v)
for k, v in agg.items(): print(f"{k:42s} n={len(v):3d} mean {sum(v)/len(v):9.1f} us  max {max(v):9.1f}")
PY
