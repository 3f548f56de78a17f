"""CPU test of the online queue policy (feedback queue + dynamic batching, §4.3) on hand traces."""
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_sched_policy_hand_traces(tmp_path):
    exe = tmp_path / "sched_policy_test"
    src = os.path.join(ROOT, "tests", "sched_policy_test.cpp")
    r = subprocess.run(["g++", "-std=c++17", "-O1", "-Wall", "-o", str(exe), src], capture_output=True, text=True)
    assert r.returncode == 0, r.stderr
    r = subprocess.run([str(exe)], capture_output=True, text=True)
    assert r.returncode == 0 and "ALL PASS" in r.stdout, r.stdout + r.stderr
