"""bench.py's own distributed skeleton at world size 2 over gloo on CPU: stream ownership
(weak and strong scaling), the timed region (barrier + synchronize on both sides, the statistics all-gather inside
it, max over ranks), the whole-job frame count, the gather latency and the one-GPU reference throughput behind the
scaling efficiency. The GPU engine is replaced by a host engine with the same interface; everything else is the
code the multi-GPU bench runs."""
import os
import socket
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
from paper_conf_icpp_zhangcjzly18_b200 import dist as fdist  # noqa: E402

NSTAT = 8


class HostEngine:
    """bench.GpuEngine's interface on the host: each step 'processes' SF frames of every owned stream and counts
    them in a per-stream statistics table the way K1 does (frames column), plus a fixed per-rank delay."""

    def __init__(self, cfg, ws, rank, delay):
        import torch
        self.torch = torch
        self.device = torch.device("cpu")
        self.sids, self.rows = bench.owned_streams(cfg, ws, rank)
        self.SF = cfg["step_frames"]
        self.frames_per_step = len(self.sids) * self.SF
        self.solo_frames_per_step = (cfg["streams"] if cfg.get("shard") else len(self.sids)) * self.SF
        self.table = torch.zeros((max(1, self.rows), NSTAT), dtype=torch.int64)
        self.delay = delay
        self.steps = 0

    def step(self, i):
        time.sleep(self.delay)
        for k, s in enumerate(self.sids):
            self.table[k, 0] += self.SF
            self.table[k, 1] += s  # a per-stream value, to check the gather's placement
        self.steps += 1

    def solo_step(self, i):
        time.sleep(self.delay)

    def join(self):
        pass

    def sync(self):
        pass

    def mark(self):
        return time.perf_counter()

    def elapsed_ms(self, t0, t1):
        return 1e3 * (t1 - t0)

    def stats(self):
        return self.table.clone()

    def start_clocks(self):
        pass

    def stop_clocks(self):
        return {"sm_mhz": None}


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, cfg_id, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        cfg = bench.CONFIGS[cfg_id]
        eng = HostEngine(cfg, world, rank, delay=0.002 * (1 + rank))  # rank 1 is the slow one
        ms, total, gathered, clk = bench.timed_region(eng, steps=5, warmup=3)
        g_us = bench.gather_us(eng, reps=5)
        fps1 = bench.solo_fps(eng, steps=3, rank=rank)
        value = total / (ms / 1e3)
        sc = bench.scaling_fields(value, fps1, world, g_us, int(gathered.shape[0]), bool(cfg.get("shard")))
        q.put((rank, eng.sids, eng.rows, ms, total, gathered.numpy(), eng.steps, fps1, sc))
    finally:
        dist.destroy_process_group()


def _run(cfg_id):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, cfg_id, q)) for r in range(2)]
    for p in procs:
        p.start()
    outs = sorted([q.get(timeout=180) for _ in procs], key=lambda t: t[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    return outs


def test_owned_streams_weak_and_strong():
    m2, m5 = bench.CONFIGS["m2"], bench.CONFIGS["m5"]
    for ws in (1, 2, 4, 8):
        weak = [bench.owned_streams(m2, ws, r) for r in range(ws)]
        assert all(rows == 30 and len(ids) == 30 for ids, rows in weak)       # fixed per-GPU work
        assert sorted(s for ids, _ in weak for s in ids) == list(range(30 * ws))
        strong = [bench.owned_streams(m5, ws, r) for r in range(ws)]
        assert sorted(s for ids, _ in strong for s in ids) == list(range(256))  # fixed total work
        assert all(rows == 256 // ws for _, rows in strong)
        for ids, _ in strong:
            assert ids == list(fdist.shard_streams(256, ws, strong.index((ids, 256 // ws))))


def test_timed_region_world2_weak():
    outs = _run("m2")
    (r0, sids0, rows0, ms0, tot0, g0, st0, f0, sc0), (r1, sids1, rows1, ms1, tot1, g1, st1, f1, sc1) = outs
    assert sids0 == list(range(30)) and sids1 == list(range(30, 60))
    # max over ranks: both ranks report the slow rank's time, which covers 5 steps of 4 ms
    assert ms0 == ms1 and ms0 >= 5 * 4.0
    # whole-job frames = 2 x one rank's (weak scaling, "frames_per_step = 2 x per-rank")
    assert tot0 == tot1 == 2 * 30 * 30 * 5
    # the gathered table holds every rank's rows in rank order: warm-up + timed steps of every stream
    for g in (g0, g1):
        assert g.shape == (60, NSTAT)
        assert np.all(g[:, 0] == 30 * 8)
        assert np.array_equal(g[:, 1], np.arange(60) * 8)
    # rank 0's solo throughput is what both ranks report; efficiency follows from it
    assert f0 == f1 > 0
    assert sc0["kind"] == "weak" and sc0["n_gpus"] == 2 and sc0["stats_gather_us"] > 0
    assert abs(sc0["efficiency"] - (tot0 / (ms0 / 1e3)) / (2 * f0)) < 1e-9


def test_timed_region_world2_strong():
    outs = _run("m5")
    (_, sids0, rows0, ms0, tot0, g0, *_r0), (_, sids1, rows1, ms1, tot1, g1, *_r1) = outs
    assert sids0 == list(range(128)) and sids1 == list(range(128, 256)) and rows0 == rows1 == 128
    assert tot0 == tot1 == 256 * 10 * 5                      # the whole stream set, split
    assert np.all(g0[:, 0] == 10 * 8) and np.array_equal(g0[:, 1], np.arange(256) * 8)
    assert _r0[-1]["kind"] == "strong"


def test_timed_region_single_process_without_group():
    """N = 1 (no process group at all): the same skeleton must run without torch.distributed initialised."""
    eng = HostEngine(bench.CONFIGS["m2"], 1, 0, delay=0.001)
    ms, total, gathered, _ = bench.timed_region(eng, steps=4, warmup=3)
    assert total == 30 * 30 * 4 and ms >= 4.0
    assert gathered.shape == (30, NSTAT) and np.all(gathered.numpy()[:, 0] == 30 * 7)
    assert bench.gather_us(eng, reps=2) >= 0
