"""GPU checks of f2 (§4.3.1): a stream re-forwarded through its image (ffsva_stream_export /
ffsva_stream_import) continues bit-identically — same distances, pass masks and logits on the same frames, its
statistics row carried over — through host and device images and across two processes (gloo handover of a host
image, both on cuda:0: the box has one GPU; the NCCL device-image path is the same calls with device tensors).
The online runtime's overload signals and detach follow the feedback-queue thresholds."""
import os
import socket

import numpy as np
import pytest

from gpu_util import Cam
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
    assert n == 256 + 30000 + 26832 + 192  # header + R + packed SNM image (bf16 FC weights) + stats row (24 x u64)
    img = cam.st.export() if where == "host" else cam.st.export(torch.empty(n, dtype=torch.uint8, device=dev))
    cam.st.close()
    st2 = ctx.import_stream(img)
    assert st2.desc.width == 640 and st2.desc.distance == ff.ffsva.DISTANCES[distance]
    assert np.array_equal(ctx.stats()[st2.slot], stats_before)  # statistics row travels with the stream
    r2 = ctx.filter_batch([(st2, d[i], i) for i in range(30)])
    _same(r1, r2)
    assert int(r1["sdd_pass"].sum()) > 0
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
    import torch
    import torch.distributed as dist
    import paper_conf_icpp_zhangcjzly18_b200 as ff
    from paper_conf_icpp_zhangcjzly18_b200 import dist as fdist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=2)
    dev = torch.device("cuda:0")
    ctx = ff.Context(dev)
    v = synth.Video(seed=95, width=640, height=360, period=6, on_len=2)
    d = torch.from_numpy(synth.frames(v, [4] * 12, list(range(12)))).to(dev)
    owned = {}
    if rank == 0:
        st = ctx.open_stream(width=640, height=360)
        st.set_reference(torch.from_numpy(synth.frames(v, [4] * 4, list(range(4)), ref=True)).to(dev))
        st.snm_load(synth.snm_weights(95, 4, bias_std=0.05))
        owned[17] = st
    before = ctx.filter_batch([(owned[17], d[i], i) for i in range(12)]) if rank == 0 else None
    reports = fdist.gather_reports(0.95 if rank == 0 else 0.1, [(17, True, 1.0)] if rank == 0 else [], 4)
    moves = fdist.plan_reforward(reports)
    fdist.reforward(moves, owned, ctx, rank)
    after = ctx.filter_batch([(owned[17], d[i], i) for i in range(12)]) if rank == 1 else None
    q.put((rank, moves, sorted(owned), before, after))
    ctx.close()
    dist.destroy_process_group()


def test_reforward_two_processes(env):
    import torch.multiprocessing as mp
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
    assert outs[0][1] == outs[1][1] == [(17, 0, 1)]
    assert outs[0][2] == [] and outs[1][2] == [17]
    _same(outs[0][3], outs[1][4])
