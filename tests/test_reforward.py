"""f2 host logic (§4.3.1): admission control and stream re-forwarding between instances —
the deterministic plan on hand cases, and (world size 2, gloo on CPU) the report all-gather and the
point-to-point image handover the GPU path runs over NCCL."""
import os
import socket

import numpy as np

from paper_conf_icpp_zhangcjzly18_b200 import dist as fdist


def test_plan_moves_overloaded_stream_to_spare_instance():
    reports = [{"busy": 0.95, "streams": [(0, False, 0.5), (1, True, 0.5)]},
               {"busy": 0.20, "streams": [(2, False, 1.0)]},
               {"busy": 0.40, "streams": [(3, False, 1.0)]}]
    assert fdist.plan_reforward(reports) == [(1, 0, 1)]  # least busy instance with spare capacity


def test_plan_spreads_several_overloaded_streams():
    # two overloaded streams, each 0.4 of a fully busy instance: the first lands on rank 1 (0.1 -> 0.5),
    # the second then prefers rank 2 (0.3 < 0.5)
    reports = [{"busy": 1.0, "streams": [(7, True, 0.4), (5, True, 0.4), (6, False, 0.2)]},
               {"busy": 0.1, "streams": []},
               {"busy": 0.3, "streams": []}]
    assert fdist.plan_reforward(reports) == [(5, 0, 1), (7, 0, 2)]


def test_plan_no_spare_capacity_no_moves():
    reports = [{"busy": 0.99, "streams": [(0, True, 1.0)]}, {"busy": 0.8, "streams": [(1, True, 1.0)]}]
    assert fdist.plan_reforward(reports, spare_busy=0.7) == []
    # the spare threshold is strict: busy == spare_busy is not spare
    assert fdist.plan_reforward([{"busy": 1.0, "streams": [(0, True, 1.0)]}, {"busy": 0.7, "streams": []}],
                                spare_busy=0.7) == []


def test_plan_never_targets_the_source_and_is_deterministic():
    rng = np.random.default_rng(3)
    for _ in range(200):
        world = int(rng.integers(1, 6))
        reports, gid = [], 0
        for r in range(world):
            k = int(rng.integers(0, 5))
            reports.append({"busy": float(rng.random()),
                            "streams": [(gid + i, bool(rng.random() < 0.4), 1.0 / max(1, k)) for i in range(k)]})
            gid += k
        m1 = fdist.plan_reforward(reports)
        assert m1 == fdist.plan_reforward(list(reversed(list(reversed(reports)))))
        owner = {g: r for r, rep in enumerate(reports) for g, _, _ in rep["streams"]}
        over = {g for rep in reports for g, o, _ in rep["streams"] if o}
        for g, src, dst in m1:
            assert src == owner[g] and dst != src and g in over
        assert len({g for g, _, _ in m1}) == len(m1)  # each stream moves at most once per round


def test_place_new_stream():
    assert fdist.place_new_stream([0.5, 0.2, 0.2]) == 1
    assert fdist.place_new_stream([0.9, 0.8]) is None
    assert fdist.place_new_stream([0.9, 0.69], spare_busy=0.7) == 1


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
        mine = [(0, rank == 0, 0.6), (1, False, 0.4)] if rank == 0 else [(2, False, 1.0)]
        reports = fdist.gather_reports(0.95 if rank == 0 else 0.3, mine, max_streams=4)
        moves = fdist.plan_reforward(reports)
        image = np.arange(64320, dtype=np.int64).astype(np.uint8) if rank == 0 else None
        got = None
        for gid, src, dst in moves:
            got = fdist.transfer_image(image, src, dst, rank)
        q.put((rank, reports, moves, None if got is None else got.numpy()))
    finally:
        dist.destroy_process_group()


def test_reports_and_image_handover_world2_gloo():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    outs = {o[0]: o for o in (q.get(timeout=120) for _ in procs)}
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in (0, 1):
        _, reports, moves, _ = outs[r]
        assert abs(reports[0]["busy"] - 0.95) < 1e-12 and abs(reports[1]["busy"] - 0.3) < 1e-12
        assert reports[0]["streams"] == [(0, True, 0.6), (1, False, 0.4)]
        assert reports[1]["streams"] == [(2, False, 1.0)]
        assert moves == [(0, 0, 1)]  # identical plan on every rank
    assert outs[0][3] is None
    assert np.array_equal(outs[1][3], np.arange(64320, dtype=np.int64).astype(np.uint8))
