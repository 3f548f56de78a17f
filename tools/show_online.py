"""Summarise the online-validation part of a bench JSON line (ladder rungs, confirmations, TOR sweep)."""
import json
import sys

d = json.load(open(sys.argv[1]))
print("value", d["value"], "frac", d["roofline"]["frac"], "validated", d.get("sustained_streams_validated"))
o = d.get("online") or {}
for k in ("sdd_snm", "sdd_snm_tyolo"):
    if k not in o:
        continue
    for tag, rs in (("rung", o[k]["rungs"]), ("confirm", o[k]["confirm"])):
        for r in rs:
            print(k, tag, r["streams"], r["seconds"], r["sustained"], "p99", round(r["latency_p99_s"], 3),
                  "decided", round(r["decided_fraction_of_window"], 4), "slope/stream",
                  round(r["backlog_slope_per_stream"], 4), "lib", r.get("library_latency"))
for t, v in o.get("online_by_tor", {}).items():
    for tag, rs in (("rung", v["rungs"]), ("confirm", v["confirm"])):
        for r in rs:
            print("tor", t, tag, r["streams"], r["seconds"], r["sustained"], "p99", round(r["latency_p99_s"], 3),
                  "decided", round(r["decided_fraction_of_window"], 4), "slope/stream",
                  round(r["backlog_slope_per_stream"], 4))
