"""GPU checks of f2 (§4.3.1): a stream re-forwarded through its image (ffsva_stream_export /
ffsva_stream_import) continues bit-identically — same distances, pass masks and logits on the same frames, its
statistics row carried over — through host and device images and across two processes (gloo handover of a host
image, both on cuda:0: the box has one GPU; the NCCL device-image path is the same calls with device tensors).
The online runtime's overload signals and detach follow the feedback-queue thresholds."""
import os
import socket

import numpy as np
import pytest

from gpu_util import Cam, check_snm, oracle_for
from synth import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    import __graft_entry__ as ge
    ge.build()
    import paper_conf_icpp_zhangcjzly18_b200 as ff
    dev = torch.device("cuda:0")
    ctx = ff.Context(dev)
    yield ff, ctx, dev
    ctx.close()


def _same(a, b):
    for k in ("ssd", "sdd_pass", "snm_pass", "snm_class", "survivor_idx"):
        assert np.array_equal(a[k], b[k]), k
    assert np.array_equal(a["logit"].view(np.uint32), b["logit"].view(np.uint32))  # bitwise, NaN included


@pytest.mark.parametrize("where", ["host", "device"])
@pytest.mark.parametrize("distance", ["mse", "nrmse", "sad"])
def test_export_import_continues_identically(env, where, distance):
    import torch
    ff, ctx, dev = env
    v = synth.Video(seed=91, width=640, height=360, period=10, on_len=4)
    delta = {"mse": 24.0, "nrmse": 0.05, "sad": 60000.0}[distance]
    cam = Cam(ctx, v, 2, dev, k_ref=4, delta=delta, distance=distance)
    host = cam.host_frames(list(range(30)))
    d = torch.from_numpy(host).to(dev)
    r1 = ctx.filter_batch([(cam.st, d[i], i) for i in range(30)])
    stats_before = ctx.stats()[cam.st.slot].copy()
    n = cam.st.image_bytes()
    assert n == 256 + 30000 + 63696 + 192  # header + R + packed SNM image (shared-memory image of K4) + stats row (24 x u64)
    img = cam.st.export() if where == "host" else cam.st.export(torch.empty(n, dtype=torch.uint8, device=dev))
    cam.st.close()
    st2 = ctx.import_stream(img)
    assert st2.desc.width == 640 and st2.desc.distance == ff.ffsva.DISTANCES[distance]
    assert np.array_equal(ctx.stats()[st2.slot], stats_before)  # statistics row travels with the stream
    r2 = ctx.filter_batch([(st2, d[i], i) for i in range(30)])
    _same(r1, r2)
    assert int(r1["sdd_pass"].sum()) > 0
    # and the continued stream against the oracle (the imported R, thresholds and SNM are the exported ones)
    want = oracle_for([(cam, host[i]) for i in range(30)])
    assert np.array_equal(r2["ssd"], want["ssd"]) and np.array_equal(r2["sdd_pass"], want["sdd_pass"])
    check_snm(r2["logit"], r2["snm_pass"], r2["snm_class"], want["logit"], [cam] * 30, want["survivors"])
    st2.close()


def test_import_rejects_garbage(env):
    ff, ctx, dev = env
    with pytest.raises(ff.ffsva.FfsvaError):
        ctx.import_stream(np.zeros(64320, np.uint8))


def test_scheduler_overload_signals_and_detach(env):
    """q_snm = 0 with every frame a target: the SNM queue goes over its threshold, the SDD stage skips the
    stream (sdd_blocked), the prefetcher is refused; detach waits for the queues, then succeeds."""
    import torch
    ff, ctx, dev = env
    from paper_conf_icpp_zhangcjzly18_b200.ffsva import Scheduler
    v = synth.Video(seed=93, width=640, height=360, period=2, on_len=2)  # every frame a target
    cam = Cam(ctx, v, 0, dev, k_ref=2)
    st = ctx.open_stream(width=640, height=360, snm_batch=1, q_sdd=1, q_snm=0)
    st.set_reference(torch.from_numpy(cam.refs).to(dev))
    st.snm_load(cam.params)
    frames = torch.from_numpy(cam.host_frames(list(range(12)))).to(dev)
    sched = Scheduler(ctx, max_frames_per_tick=64, snm_slots=64)
    acc = sched.push([(st, frames[i], i) for i in range(6)])
    assert acc.tolist() == [1, 1, 0, 0, 0, 0]          # SDD queue over q_sdd = 1 after two frames
    sched.tick()                                        # both pass SDD: SNM depth 2 -> 1 after a pop of 1
    sched.push([(st, frames[i], i) for i in range(2, 4)])
    sched.tick()                                        # SNM depth 1 > q_snm = 0: SDD skips the stream
    load = sched.stream_load(st, reset=True)
    assert load["refused"] >= 4 and load["sdd_blocked"] >= 1 and load["max_sdd"] >= 2
    assert sched.stream_load(st)["refused"] == 0       # counters were reset
    assert not sched.detach(st)                         # frames still queued
    for _ in range(20):
        sched.tick()
        if sched.detach(st):
            break
    else:
        raise AssertionError("stream never detached")
    assert sched.stream_load(st)["pushed"] == 0         # detached: idle
    assert sched.push([(st, frames[5], 5)]).tolist() == [1]  # re-attaches on push
    sched.destroy()
    st.close()
    cam.st.close()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _proc(rank, port, q):
    """One instance of the f2 controller test (both processes on cuda:0, gloo: the box has one GPU; with NCCL the
    same calls move the image as a device tensor)."""
    import torch
    import torch.distributed as dist
    import paper_conf_icpp_zhangcjzly18_b200 as ff
    from paper_conf_icpp_zhangcjzly18_b200.online import run_controlled
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=2)
    dev = torch.device("cuda:0")
    ctx = ff.Context(dev)
    v = synth.Video(seed=95, width=640, height=360, period=2, on_len=2)  # every frame holds a target
    NF = 12
    content = {g: torch.from_numpy(synth.frames(v, [g] * NF, list(range(NF)))).to(dev) for g in range(3)}
    owned = {}
    for g in ((0, 1) if rank == 0 else (2,)):
        # camera 0 (300 frames/s, every frame a target, BatchSize 1) overloads rank 0: its SNM queue goes over q_snm
        st = ctx.open_stream(width=640, height=360, snm_batch=1 if g == 0 else 30, q_snm=2 if g == 0 else 10)
        st.set_reference(torch.from_numpy(synth.frames(v, [g] * 4, list(range(4)), ref=True)).to(dev))
        st.snm_load(synth.snm_weights(95, g, bias_std=0.05))
        owned[g] = st
    ctx.stats(reset=True)
    out = run_controlled(ctx, owned, content, NF, 3, seconds=5.0, spare_fps=45.0, interval_s=1.0, window_s=2.0,
                         fps={0: 300.0, 1: 30.0, 2: 30.0})
    stats = ctx.stats()
    rows = {g: stats[st.slot].copy() for g, st in owned.items()}
    q.put((rank, out["history"], out["owned"], {g: sorted(d) for g, d in out["decided"].items()},
           {g: {k: (int(r["ssd"]), int(r["sdd_pass"]), float(r["logit"])) for k, r in d.items()}
            for g, d in out["decided"].items()}, rows))
    for st in owned.values():
        st.close()
    ctx.close()
    dist.destroy_process_group()


def test_reforward_controller_two_processes(env):
    """f2 in the online loop: rank 0 runs cameras 0 (300 frames/s) and 1 (30 frames/s) with
    camera 0 overloading its SNM queue; rank 1 runs camera 2 at 30 frames/s, below the 45 frames/s spare level for
    the whole 2-s window. The controller re-forwards camera 0 to rank 1, which continues it from the frame rank 0 reached; the
    frames each side decided agree with the oracle; the stream's statistics row travels with it."""
    import torch.multiprocessing as mp
    from oracle import oracle as orc
    mctx = mp.get_context("spawn")
    q = mctx.Queue()
    port = _free_port()
    procs = [mctx.Process(target=_proc, args=(r, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    outs = {o[0]: o for o in (q.get(timeout=300) for _ in procs)}
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    moves = [m for h in outs[0][1] for m in h["moves"]]
    assert moves == [(0, 0, 1)], outs[0][1] and [m for h in outs[1][1] for m in h["moves"]] == moves
    assert outs[0][2] == [1] and outs[1][2] == [0, 2]
    f0, f1 = outs[0][3].get(0, []), outs[1][3].get(0, [])
    assert f0 and f1 and max(f0) < min(f1), "rank 1 continues camera 0 after the frames rank 0 decided"
    assert set(f0) | set(f1) == set(range(max(f1) + 1)), "no frame of camera 0 lost in the handover"
    # statistics row: the imported stream continued rank 0's counters
    assert int(outs[1][5][0][0]) == len(f0) + len(f1)
    # every decided frame of camera 0 (either side) against the oracle
    v = synth.Video(seed=95, width=640, height=360, period=2, on_len=2)
    R = orc.reference(synth.frames(v, [0] * 4, list(range(4)), ref=True), 640, 100, 100)
    params = synth.snm_weights(95, 0, bias_std=0.05)
    for side in (0, 1):
        for k, (ssd, sp, lg) in list(outs[side][4][0].items())[::7]:
            w = orc.filter_frames([synth.frame(v, 0, k % 12)], 640, [R], [24.0], [params], [np.float32(0.2)],
                                  [np.float32(0.8)], [np.float32(0.5)])
            assert ssd == int(w["ssd"][0]) and sp == int(w["sdd_pass"][0]) == 1
            assert abs(lg - w["logit"][0]) <= 2e-2
