"""Small run through every kernel path (K1 bulk + stream variants, K2, K3, K4, reference, T-YOLO view kernels, online
scheduler in synchronous and pipelined mode) for
compute-sanitizer (memcheck / racecheck / synccheck / initcheck). Prints OK at the end."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_zhangcjzly18_b200 as ff  # noqa: E402
from paper_conf_icpp_zhangcjzly18_b200.ffsva import Scheduler  # noqa: E402
from synth import synth  # noqa: E402


def minimal():
    """--minimal (racecheck to completion): the narrow-row K1 (warp-segment pipeline), K3 and K4 on 8 frames of two
    streams, the one-CTA-per-band K1 on 2 small frames, the CTA-pair K1 on one 720p frame, and two synchronous
    scheduler ticks."""
    dev = torch.device("cuda:0")
    ctx = ff.Context(dev)
    v = synth.Video(seed=5, width=640, height=360, period=4, on_len=2)
    streams = []
    for s in range(2):
        st = ctx.open_stream(width=640, height=360, delta_diff=0.0 if s else 24.0, snm_batch=2)
        st.set_reference(torch.from_numpy(synth.frames(v, [s] * 2, [0, 1], ref=True)).to(dev))
        st.snm_load(synth.snm_weights(5, s, bias_std=0.1))
        streams.append(st)
    d = torch.from_numpy(synth.frames(v, [0, 1] * 4, [0, 0, 1, 1, 2, 2, 3, 3])).to(dev)
    items = [(streams[i % 2], d[i], i) for i in range(8)]
    r = ctx.filter_batch(items)
    assert int(r["sdd_pass"][1::2].sum()) == 4  # delta 0: every frame of stream 1 reaches K4
    for (W, H, n) in ((128, 100, 2), (1280, 720, 1)):
        vb = synth.Video(seed=6, width=W, height=H, period=4, on_len=2)
        sb = ctx.open_stream(width=W, height=H, delta_diff=0.0, snm_batch=2)
        sb.set_reference(torch.from_numpy(synth.frames(vb, [0], [0], ref=True)).to(dev))
        sb.snm_load(synth.snm_weights(6, 0))
        db = torch.from_numpy(synth.frames(vb, [0] * n, list(range(n)))).to(dev)
        ctx.filter_batch([(sb, db[i], i) for i in range(n)])
        sb.close()
    sched = Scheduler(ctx, max_frames_per_tick=8, snm_slots=16)
    sched.push(items)
    for _ in range(2):
        sched.tick()
    sched.destroy()
    ctx.close()
    torch.cuda.synchronize()
    print("OK (minimal)")


def main():
    if "--minimal" in sys.argv:
        return minimal()
    dev = torch.device("cuda:0")
    ctx = ff.Context(dev)
    v = synth.Video(seed=5, width=640, height=360, period=4, on_len=2)
    streams = []
    for s in range(2):
        st = ctx.open_stream(width=640, height=360, snm_batch=2, q_sdd=2, q_snm=3)
        st.set_reference(torch.from_numpy(synth.frames(v, [s] * 2, [0, 1], ref=True)).to(dev))
        st.snm_load(synth.snm_weights(5, s, bias_std=0.1))
        streams.append(st)
    host = synth.frames(v, [0, 1] * 4, [0, 0, 1, 1, 2, 2, 3, 3])
    d = torch.from_numpy(host).to(dev)
    items = [(streams[i % 2], d[i], i) for i in range(8)]
    r1 = ctx.filter_batch(items)
    os.environ["FFSVA_SDD_KERNEL"] = "stream"
    r2 = ctx.filter_batch(items)
    del os.environ["FFSVA_SDD_KERNEL"]
    assert np.array_equal(r1["ssd"], r2["ssd"])
    pb = ctx.prepare(items)
    s = torch.cuda.Stream()
    pb.launch(s)
    pb.launch(s)
    r3 = pb.fetch(s)
    assert np.array_equal(r1["ssd"], r3["ssd"])
    pb.destroy()
    pinned = [torch.from_numpy(h).pin_memory() for h in host]
    r4 = ctx.filter_batch([(streams[i % 2], pinned[i].data_ptr(), i) for i in range(8)], host=True)
    assert np.array_equal(r1["ssd"], r4["ssd"])
    # the 256- and 384-thread K1 block sizes (720p and 1080p rows); racecheck (--no-tyolo) takes 1 frame each
    no_ty = "--no-tyolo" in sys.argv
    for (W, H) in ((1280, 720), (1920, 1080)):
        vb = synth.Video(seed=6, width=W, height=H, period=4, on_len=2)
        sb = ctx.open_stream(width=W, height=H, snm_batch=2)
        sb.set_reference(torch.from_numpy(synth.frames(vb, [0], [0], ref=True)).to(dev))
        sb.snm_load(synth.snm_weights(6, 0))
        nb = 1 if no_ty else 3
        db = torch.from_numpy(synth.frames(vb, [0] * nb, list(range(nb)))).to(dev)
        rb = ctx.filter_batch([(sb, db[i], i) for i in range(nb)])
        assert int(rb["sdd_pass"].sum()) == sum(int(synth.is_target(vb, 0, t)) for t in range(nb))
        sb.close()
    # f3 variants: SAD + previous-frame reference (K2 / K2b) and NRMSE, mixed in one batch
    extra = []
    for s_id, (dist, mode) in enumerate([("sad", "previous"), ("nrmse", "background")]):
        st = ctx.open_stream(width=640, height=360, delta_diff=0.01 if dist == "nrmse" else 1000.0,
                             distance=dist, ref_mode=mode)
        st.set_reference(torch.from_numpy(synth.frames(v, [s_id] * 2, [0, 1], ref=True)).to(dev))
        st.snm_load(synth.snm_weights(5, s_id))
        extra.append(st)
    r5 = ctx.filter_batch([(extra[i % 2], d[i], i) for i in range(8)] + items)
    assert np.array_equal(r5["ssd"][8:], r1["ssd"])
    for st in extra:
        st.close()
    # T-YOLO stage (f1): standalone on 3 frames, then attached to the online runtime (three-stage cascade).
    # --no-tyolo (racecheck: its shared-memory tracking of the T-YOLO GEMMs does not finish in the time limit)
    # keeps the SDD -> SNM cascade only.
    if no_ty:
        sched = Scheduler(ctx, max_frames_per_tick=4, snm_slots=16)
        sched.set_pipeline(True)
        for t in range(6):
            if t < 4:
                sched.push([(streams[i % 2], d[i], i) for i in range(8)])
            sched.tick(s)
        sched.destroy()
        ctx.close()
        torch.cuda.synchronize()
        print("OK (without T-YOLO)")
        return
    ty = ff.Tyolo(ctx, synth.tyolo_weights(5))
    r6 = ty.run([(streams[i % 2], d[i], i) for i in range(3)], raw=True)
    assert r6["counts"].shape == (3,)
    sched = Scheduler(ctx, max_frames_per_tick=4, snm_slots=8)
    sched.set_tyolo(ty, num_tyolo=1)
    for t in range(6):
        sched.push([(streams[i % 2], d[i], i) for i in range(8)])
        sched.tick(s)
    sched.destroy()
    # pipelined ticks (ffsva_sched_set_pipeline): kernels of cycle k overlap the host half of cycle k + 1
    sched = Scheduler(ctx, max_frames_per_tick=4, snm_slots=16)
    sched.set_pipeline(True)
    for t in range(8):
        if t < 6:
            sched.push([(streams[i % 2], d[i], i) for i in range(8)])
        sched.tick(s)
    sched.destroy()
    ty.destroy()
    ctx.close()
    torch.cuda.synchronize()
    print("OK")


if __name__ == "__main__":
    main()
