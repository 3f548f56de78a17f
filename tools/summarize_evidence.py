"""Turn the gpurun_out/ evidence of tools/evidence.sh into tracked summaries under profiles/<round>/.

  python tools/summarize_evidence.py r01

Writes:
  profiles/<round>/launches_<cfg>.csv   the ncu launch list (gpu__time_duration.sum per launch, cold, serialised)
  profiles/<round>/launches_<cfg>.md    per-kernel mean time and share of the step from that list
  profiles/<round>/ncu_full_<name>.json key metrics of each `ncu --set full` capture (tools/ncu_summary.py)
  profiles/ncu_k1_traffic.json          dram read+write bytes per K1 launch, per config (bench.py's `traffic`)
  profiles/<round>/{bench.json,pytest_gpu.log,smoke.log,sanitize_*.log} copies
"""
import csv
import glob
import io
import json
import os
import re
import shutil
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
from ncu_summary import summarize  # noqa: E402

OUT = os.path.join(ROOT, "gpurun_out")


def short(name):
    for k, v in (("tyolo_conv", "K5 tyolo_conv"), ("tyolo_resize", "K5 tyolo_resize"), ("tyolo_pool", "K5 tyolo_pool_s1"),
                 ("tyolo_l1", "K5a tyolo_l1"), ("tyolo_l2", "K5b tyolo_l2"), ("tyolo_pslab", "K5c tyolo_pslab"),
                 ("tyolo_slab", "K5d tyolo_slab"),
                 ("sdd_prev", "K2 sdd_prev"), ("ref_update", "K2b ref_update"), ("sdd", "K1 sdd"),
                 ("compact", "K3 compact"), ("snm", "K4 snm")):
        if k in name:
            return v
    return name[:40]


def launch_table(path):
    with open(path) as f:
        text = f.read()
    # ncu prefixes the CSV with ==PROF== lines; keep from the header on
    i = text.find('"ID"')
    rows = list(csv.DictReader(io.StringIO(text[i:])))
    per = {}
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", ""))
        unit = r.get("Metric Unit", "ns")
        us = v / 1000.0 if unit == "ns" else (v if unit == "us" else v * 1000.0 if unit == "ms" else v)
        per.setdefault(short(r["Kernel Name"]), []).append(us)
    total = sum(sum(v) for v in per.values())
    lines = ["| kernel | launches | mean µs | median µs | share of summed time |", "|---|---|---|---|---|"]
    for k, v in sorted(per.items()):
        lines.append(f"| {k} | {len(v)} | {statistics.mean(v):.1f} | {statistics.median(v):.1f} | "
                     f"{sum(v) / total:.3f} |")
    return "\n".join(lines), per


def main():
    rnd = sys.argv[1] if len(sys.argv) > 1 else "r01"
    dst = os.path.join(ROOT, "profiles", rnd)
    os.makedirs(dst, exist_ok=True)
    for f in ["bench.json", "bench.err", "bench_reference.json", "tyolo_profile.json", "tyolo_profile.log",
              "pytest_gpu.log", "smoke.log", "nvidia-smi.txt"] + \
            [os.path.basename(p) for p in glob.glob(os.path.join(OUT, "sanitize_*.log"))] + \
            [os.path.basename(p) for p in glob.glob(os.path.join(OUT, "bench_*.json"))]:
        p = os.path.join(OUT, f)
        if os.path.exists(p):
            shutil.copy(p, os.path.join(dst, f))
    for p in glob.glob(os.path.join(OUT, "launches_*.csv")):
        cfg = re.sub(r"^launches_|\.csv$", "", os.path.basename(p))
        shutil.copy(p, os.path.join(dst, os.path.basename(p)))
        table, _ = launch_table(p)
        with open(os.path.join(dst, f"launches_{cfg}.md"), "w") as f:
            f.write(f"# ncu launch list, config {cfg} (gpu__time_duration.sum, --clock-control none; "
                    "cold-cache and serialised: compare shares, not absolutes)\n\n" + table + "\n")
        print(cfg, "\n" + table)
    tpath = os.path.join(ROOT, "profiles", "ncu_k1_traffic.json")
    traffic = json.load(open(tpath)) if os.path.exists(tpath) else {}
    for p in glob.glob(os.path.join(OUT, "*.ncu-rep")):
        name = re.sub(r"^prof_|\.ncu-rep$", "", os.path.basename(p))
        res = summarize(p)
        with open(os.path.join(dst, f"ncu_full_{name}.json"), "w") as f:
            json.dump(res, f, indent=1)
        print(name, json.dumps(res[0] if res else {}, indent=1))
        m = re.match(r"k1_(\w+)", name)
        if m and res:
            def to_bytes(s):
                v, *u = s.split()
                scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}
                return float(v.replace(",", "")) * scale.get(u[0] if u else "byte", 1)
            b = [to_bytes(d["dram__bytes_read.sum"]) + to_bytes(d["dram__bytes_write.sum"]) for d in res
                 if "dram__bytes_read.sum" in d]
            if b:
                traffic[m.group(1)] = sum(b) / len(b)
    with open(tpath, "w") as f:
        json.dump(traffic, f, indent=1)
    print("traffic", traffic)


if __name__ == "__main__":
    main()
