"""Host-side pieces of bench.py that run without a GPU: the CPU-oracle baseline worker (one core of the multi-core
figure) and the config table against BASELINE.json's workloads."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def test_oracle_worker_runs_the_unchanged_oracle():
    cfg = bench.CONFIGS["m1"]
    n, dt = bench._oracle_worker((cfg, 0, 0, 2))
    assert n == 2 and dt > 0


def test_configs_cover_baseline_workloads():
    base = json.load(open(os.path.join(ROOT, "BASELINE.json")))
    assert len(base["configs"]) == 5
    c = bench.CONFIGS
    assert (c["m1"]["W"], c["m1"]["H"], c["m1"]["streams"], c["m1"]["pool_frames"]) == (640, 360, 1, 300)
    assert (c["m2"]["W"], c["m2"]["H"], c["m2"]["streams"]) == (1280, 720, 30)
    assert (c["m3"]["W"], c["m3"]["H"], c["m3"]["streams"]) == (1920, 1080, 1)
    assert {c[k]["on_len"] * 100 // c[k]["period"] for k in ("m4_1", "m4_10", "m4_50")} == {1, 10, 50}
    assert all(c[k]["streams"] == 64 for k in ("m4_1", "m4_10", "m4_50"))
    assert (c["m5"]["W"], c["m5"]["H"], c["m5"]["streams"], c["m5"].get("shard")) == (1920, 1080, 256, True)


def test_cpu_model_string():
    assert isinstance(bench._cpu_model(), str) and bench._cpu_model()
