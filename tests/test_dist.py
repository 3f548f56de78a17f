"""Multi-process (world size 2, gloo on CPU) checks of the stream-sharding and statistics-gather logic the
multi-GPU bench uses with NCCL."""
import os
import socket

import numpy as np
import pytest

from paper_conf_icpp_zhangcjzly18_b200 import dist as fdist


def test_shard_streams_partition():
    for n in [1, 7, 30, 256, 257]:
        for world in [1, 2, 3, 4, 8]:
            owned = [list(fdist.shard_streams(n, world, r)) for r in range(world)]
            flat = [s for o in owned for s in o]
            assert flat == list(range(n))                         # contiguous, disjoint, complete
            assert max(map(len, owned)) - min(map(len, owned)) <= 1  # balanced
            for r, o in enumerate(owned):
                for s in o:
                    assert fdist.owner_of(s, n, world) == r


def test_summarize():
    st = np.zeros((3, 24), np.int64)
    st[:, 0] = [30, 30, 30]
    st[:, 1] = [3, 0, 6]
    st[:, 2] = [1, 0, 3]
    st[:, 3] = [30000 * 10, 0, 0]
    st[:, 7] = [1, 0, 1]
    s = fdist.summarize(st)
    assert s["frames"] == 90 and s["sdd_pass"] == 9 and s["snm_pass"] == 4
    assert abs(s["sdd_pass_ratio"] - 0.1) < 1e-12 and abs(s["snm_pass_ratio"] - 4 / 9) < 1e-12
    assert abs(s["mean_mse"] - 10 / 90) < 1e-12
    assert s["snm_batches"] == 2
    # latency columns (include/ffsva.h: 8 decided, 9 sum us, 10.. bins; bin 0 < 1 ms, bin k in [2^(k-1), 2^k) ms)
    st[0, 8], st[0, 9], st[0, 10 + 0], st[0, 10 + 3] = 4, 3 * 500 + 5000, 3, 1   # 3 x 0.5 ms + 1 x 5 ms
    s = fdist.summarize(st)
    assert s["decided"] == 4 and abs(s["latency_mean_ms"] - 6.5 / 4) < 1e-12
    assert s["latency_p50_ms_le"] == 1.0 and s["latency_p99_ms_le"] == 8.0


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        n = 7
        mine = list(fdist.shard_streams(n, world, rank))
        rows = max(len(list(fdist.shard_streams(n, world, r))) for r in range(world))
        local = torch.full((rows, 8), -1, dtype=torch.int64)
        for i, s in enumerate(mine):
            local[i] = torch.arange(8) + 100 * s     # stream s's counters
        g = fdist.gather_stats(local)
        # max-over-ranks timing reduction used by bench.py
        t = torch.tensor([1.0 + rank], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        q.put((rank, g.numpy(), float(t.item())))
    finally:
        dist.destroy_process_group()


def test_gather_stats_world2_gloo():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    outs = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, g, tmax in outs:
        assert tmax == 2.0
        rows = g.shape[0] // 2
        streams = [s for r in range(2) for s in fdist.shard_streams(7, 2, r)]
        got = [g[r * rows + i] for r in range(2) for i in range(len(list(fdist.shard_streams(7, 2, r))))]
        for s, row in zip(streams, got):
            assert np.array_equal(row, np.arange(8) + 100 * s)
