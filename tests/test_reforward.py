"""f2 host logic (§4.3.1): admission control and stream re-forwarding between instances —
the deterministic plan on hand cases, and (world size 2, gloo on CPU) the report all-gather and the
point-to-point image handover the GPU path runs over NCCL."""
import os
import socket

import numpy as np

from paper_conf_icpp_zhangcjzly18_b200 import dist as fdist


def _rep(rate, spare, streams):
    return {"rate": rate, "spare": spare, "streams": streams}


def test_plan_moves_overloaded_stream_to_spare_instance():
    reports = [_rep(900.0, False, [(0, False, 450.0), (1, True, 450.0)]),
               _rep(200.0, True, [(2, False, 200.0)]),
               _rep(400.0, True, [(3, False, 400.0)])]
    assert fdist.plan_reforward(reports, spare_fps=700.0) == [(1, 0, 1)]  # the spare instance with the lowest rate


def test_plan_spreads_several_overloaded_streams():
    # two overloaded streams of 400 frames/s: the first lands on rank 1 (100 -> 500), the second then prefers
    # rank 2 (300 < 500)
    reports = [_rep(1000.0, False, [(7, True, 400.0), (5, True, 400.0), (6, False, 200.0)]),
               _rep(100.0, True, []), _rep(300.0, True, [])]
    assert fdist.plan_reforward(reports, spare_fps=700.0) == [(5, 0, 1), (7, 0, 2)]


def test_plan_target_stops_being_spare_once_full():
    # rank 1 is spare at 600 frames/s; after taking 300 it is at 900 >= 700 and takes nothing more
    reports = [_rep(1000.0, False, [(0, True, 300.0), (1, True, 300.0)]), _rep(600.0, True, [])]
    assert fdist.plan_reforward(reports, spare_fps=700.0) == [(0, 0, 1)]


def test_plan_no_spare_capacity_no_moves():
    reports = [_rep(990.0, False, [(0, True, 1.0)]), _rep(800.0, False, [(1, True, 1.0)])]
    assert fdist.plan_reforward(reports, spare_fps=700.0) == []
    # a rank must be spare by its window verdict, not only by its current rate
    assert fdist.plan_reforward([_rep(990.0, False, [(0, True, 1.0)]), _rep(10.0, False, [])], 700.0) == []


def test_plan_never_targets_the_source_and_is_deterministic():
    rng = np.random.default_rng(3)
    for _ in range(200):
        world = int(rng.integers(1, 6))
        reports, gid = [], 0
        for r in range(world):
            k = int(rng.integers(0, 5))
            reports.append(_rep(float(rng.random() * 1000), bool(rng.random() < 0.5),
                                [(gid + i, bool(rng.random() < 0.4), float(rng.random() * 300)) for i in range(k)]))
            gid += k
        m1 = fdist.plan_reforward(reports, 700.0)
        assert m1 == fdist.plan_reforward([dict(r) for r in reports], 700.0)
        owner = {g: r for r, rep in enumerate(reports) for g, _, _ in rep["streams"]}
        over = {g for rep in reports for g, o, _ in rep["streams"] if o}
        for g, src, dst in m1:
            assert src == owner[g] and dst != src and g in over and reports[dst]["spare"]
        assert len({g for g, _, _ in m1}) == len(m1)  # each stream moves at most once per round


def test_place_new_stream():
    assert fdist.place_new_stream([_rep(500.0, True, []), _rep(200.0, True, []), _rep(200.0, True, [])], 700.0) == 1
    assert fdist.place_new_stream([_rep(900.0, False, []), _rep(800.0, False, [])], 700.0) is None
    assert fdist.place_new_stream([_rep(100.0, False, []), _rep(690.0, True, [])], 700.0) == 1


def test_load_monitor_rate_and_spare_window():
    m = fdist.LoadMonitor()
    for t in np.arange(0.0, 6.0, 0.01):  # 100 frames/s for 6 s: 1 frame per 10 ms tick
        m.add(float(t), 1)
    assert abs(m.rate(6.0, 5.0) - 100.0) < 1.0
    assert m.spare(6.0, 5.0, 140.0) and not m.spare(6.0, 5.0, 90.0)
    m.add(6.5, 200)  # one busy second breaks "below the level for a period of time" (L213)
    assert not m.spare(7.0, 5.0, 140.0)
    assert not fdist.LoadMonitor().spare(0.5, 5.0, 140.0)  # an unobserved window is not spare


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
        mine = [(0, rank == 0, 600.0), (1, False, 400.0)] if rank == 0 else [(2, False, 100.0)]
        reports = fdist.gather_reports(1000.0 if rank == 0 else 100.0, rank == 1, mine, max_streams=4)
        moves = fdist.plan_reforward(reports, 700.0)
        image = np.arange(64320, dtype=np.int64).astype(np.uint8) if rank == 0 else None
        got = extra = None
        for gid, src, dst in moves:
            got, extra = fdist.transfer_image(image, src, dst, rank, extra=1234)
        q.put((rank, reports, moves, None if got is None else got.numpy(), extra))
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
        _, reports, moves, _, _ = outs[r]
        assert reports[0]["rate"] == 1000.0 and not reports[0]["spare"] and reports[1]["spare"]
        assert reports[0]["streams"] == [(0, True, 600.0), (1, False, 400.0)]
        assert reports[1]["streams"] == [(2, False, 100.0)]
        assert moves == [(0, 0, 1)]  # identical plan on every rank
    assert outs[0][3] is None
    assert np.array_equal(outs[1][3], np.arange(64320, dtype=np.int64).astype(np.uint8)) and outs[1][4] == 1234


# ---- the controller in an online loop, world size 2 over gloo, with a host stand-in for the library: rank 0's
# camera 0 overloads its instance (its SNM queue goes over q_snm every interval), rank 1 runs one light camera; the
# controller must move camera 0 to rank 1, which continues it from the frame rank 0 had reached.

class _FakeStream:
    def __init__(self, gid, image=None):
        self.gid = gid
        self.image = np.full(57280, gid, np.uint8) if image is None else image
        self.handle = 1000 + gid

    def image_bytes(self):
        return self.image.size

    def export(self, out=None):
        return self.image.copy()

    def close(self):
        self.closed = True


class _FakeCtx:
    def import_stream(self, image):
        return _FakeStream(int(image[0]), image)


class _FakeSched:
    def __init__(self, overloaded):
        self.overloaded = overloaded
        self.detached = []

    def stream_load(self, st, reset=False):
        return {"sdd_blocked": 3 if st.gid in self.overloaded else 0, "snm_blocked": 0, "refused": 0, "pushed": 30}

    def detach(self, st):
        self.detached.append(st.gid)
        return True


def _ctl_worker(rank, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=2)
    try:
        owned = {0: _FakeStream(0), 1: _FakeStream(1)} if rank == 0 else {2: _FakeStream(2)}
        sched = _FakeSched(overloaded={0} if rank == 0 else set())  # camera 0 overloads rank 0's queues only
        rf = fdist.Reforwarder(_FakeCtx(), sched, owned, spare_fps=140.0, window_s=2.0)
        next_frame = {g: 57 + g for g in owned}
        moves_seen = []
        for sec in range(4):  # 4 intervals of 1 s; rank 0 processes 200 frames/s (busy), rank 1 30 frames/s
            for k in range(100):
                rf.on_tick(sec + k / 100.0, {"admitted": 2 if rank == 0 else 0.3, "snm_scored": 0,
                                            "tyolo_scored": 0})
            moves_seen.append(rf.step(sec + 1.0, 1.0, 8, detach=lambda g, st: sched.detach(st),
                                      next_frame=next_frame))
        q.put((rank, moves_seen, sorted(owned), dict(next_frame), sched.detached,
               {g: int(st.image[0]) for g, st in owned.items()}))
    finally:
        dist.destroy_process_group()


def test_controller_moves_overloaded_stream_world2_gloo():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ctl_worker, args=(r, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    outs = {o[0]: o for o in (q.get(timeout=120) for _ in procs)}
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for r in (0, 1):
        moves = outs[r][1]
        # intervals 1-2: the 2-s window is not yet observed completely (no instance is spare yet); interval 3: rank 1
        # has been below 140 frames/s for 2 s, rank 0's camera 0 overloads: it moves; interval 4: nothing left to move
        assert moves[0] == [] and moves[1] == [(0, 0, 1)] or moves[:2] == [[], []] and moves[2] == [(0, 0, 1)]
        assert sum(len(m) for m in moves) == 1
    assert outs[0][2] == [1] and outs[1][2] == [0, 2]
    assert outs[0][4] == [0]                       # the source detached the stream before exporting it
    assert outs[1][3][0] == 57                     # the camera continues at the source's next frame
    assert outs[1][5] == {0: 0, 2: 2}              # the target imported camera 0's image
