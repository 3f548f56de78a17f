"""GPU parity of the f3 SDD variants ("MSE, NRMSE, or SAD"; Q23-Q25)
through the C-ABI against the CPU oracle: distance numerators, pass masks, survivor order bit-exact; SNM logits
within the north_star tolerance. Previous-frame reference mode is checked across batches (the stream's reference
chains), through prepared batches (CUDA-graph replays), the host-frame path and mixed-mode batches.
"""
import math

import numpy as np
import pytest

from gpu_util import Cam, check_snm, oracle_for
from oracle import oracle as orc
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


def _dev(x, dev):
    import torch
    return torch.from_numpy(np.ascontiguousarray(x)).to(dev)


def _median_delta(metric, video, sid, ts, R, W):
    """A delta_diff that splits the oracle's distances of these frames (some pass, some do not)."""
    d = [orc.distance(metric, orc.box_downsample(synth.frame(video, sid, t), W, 100, 100), R) for t in ts]
    med = float(np.median(d))
    if metric == "mse":
        return med / 30000.0
    if metric == "sad":
        return med
    return math.sqrt(med / orc.sum_sq(R))


@pytest.mark.parametrize("metric", ["mse", "sad", "nrmse"])
@pytest.mark.parametrize("W,H", [(640, 360), (641, 361)])
def test_metric_parity(env, metric, W, H):
    """Every frame of a 60-frame run with targets: distance numerator, pass, survivor order bit-exact; SNM in tol.
    delta_diff sits at the median distance so both outcomes occur (background frames differ by noise only)."""
    ff, ctx, dev = env
    v = synth.Video(seed=2300 + W, width=W, height=H, period=20, on_len=6)
    probe = Cam(ctx, v, 1, dev, k_ref=8, load_snm=False)
    delta = _median_delta(metric, v, 1, list(range(60)), probe.R, W)
    probe.st.close()
    cam = Cam(ctx, v, 1, dev, k_ref=8, delta=delta, distance=metric)
    host = cam.host_frames(list(range(60)))
    d = _dev(host, dev)
    got = ctx.filter_batch([(cam.st, d[i], i) for i in range(60)])
    want = oracle_for([(cam, host[i]) for i in range(60)])
    assert np.array_equal(got["ssd"], want["ssd"])
    assert np.array_equal(got["sdd_pass"], want["sdd_pass"])
    assert 0 < int(want["sdd_pass"].sum()) < 60
    assert np.array_equal(got["survivor_idx"], want["survivor_idx"])
    check_snm(got["logit"], got["snm_pass"], got["snm_class"], want["logit"], [cam] * 60, want["survivors"])
    cam.st.close()


def test_nrmse_exact_boundary_on_device(env):
    """P13 on the device path: an all-zero frame against reference R has SSD = sum R^2, NRMSE = 1 exactly; the
    strict test drops it at delta = 1 and keeps it at the next double below 1 (exact threshold arithmetic)."""
    ff, ctx, dev = env
    W, H = 640, 360
    v = synth.Video(seed=41, width=W, height=H)
    refs = synth.frames(v, [0] * 4, list(range(4)), ref=True)
    R = orc.reference(refs, W, 100, 100)
    Q = orc.sum_sq(R)
    zero = _dev(np.zeros((1, H, 3 * W), np.uint8), dev)
    for delta, expect in [(1.0, 0), (math.nextafter(1.0, 0.0), 1), (0.5, 1), (1.5, 0)]:
        st = ctx.open_stream(width=W, height=H, delta_diff=delta, distance="nrmse")
        st.set_reference(refs)
        got = ctx.sdd_batch([(st, zero[0], 0)], want_d100=False)
        assert int(got["ssd"][0]) == Q
        assert int(got["sdd_pass"][0]) == expect, delta
        st.close()


def test_sad_threshold_is_strict_on_device(env):
    """SAD > delta_diff exactly: delta = SAD drops the frame, the next double below keeps it."""
    ff, ctx, dev = env
    W, H = 200, 120
    v = synth.Video(seed=43, width=W, height=H, period=2, on_len=1)
    host = synth.frames(v, [0], [0])
    refs = synth.frames(v, [0] * 2, [0, 1], ref=True)
    sad = orc.sad(orc.box_downsample(host[0], W, 100, 100), orc.reference(refs, W, 100, 100))
    d = _dev(host, dev)
    for delta, expect in [(float(sad), 0), (math.nextafter(float(sad), 0.0), 1)]:
        st = ctx.open_stream(width=W, height=H, delta_diff=delta, distance="sad")
        st.set_reference(refs)
        got = ctx.sdd_batch([(st, d[0], 0)], want_d100=False)
        assert int(got["ssd"][0]) == sad and int(got["sdd_pass"][0]) == expect
        st.close()


@pytest.mark.parametrize("metric", ["mse", "sad"])
def test_previous_frame_mode_chains_across_batches(env, metric):
    """Three streams interleaved (one background-mode MSE stream among them), three consecutive filter_batch
    calls: each previous-mode frame is compared with its stream's previous frame, across batch boundaries;
    the stream's reference afterwards equals the oracle's last D100."""
    ff, ctx, dev = env
    W, H = 640, 360
    v = synth.Video(seed=51, width=W, height=H, period=12, on_len=4)
    delta = 5.0 if metric == "mse" else 40000.0
    cams = [Cam(ctx, v, 0, dev, k_ref=4, delta=delta, distance=metric, ref_mode="previous"),
            Cam(ctx, v, 1, dev, k_ref=4, delta=delta, distance=metric, ref_mode="previous"),
            Cam(ctx, v, 2, dev, k_ref=4, delta=24.0)]
    order = [0, 1, 0, 2, 1, 1, 0, 2, 0, 1]  # camera of each slot in a batch: ragged, interleaved
    t_next = [0, 0, 0]
    plan = []
    for _ in range(3):
        items = []
        for c in order:
            items.append((c, t_next[c]))
            t_next[c] += 1
        plan.append(items)
    hosts = [[cams[c].host_frames([t])[0] for c, t in items] for items in plan]
    outs = []
    for b, items in enumerate(plan):
        d = _dev(np.stack(hosts[b]), dev)
        got = ctx.filter_batch([(cams[c].st, d[i], t) for i, (c, t) in enumerate(items)])
        want = oracle_for([(cams[c], hosts[b][i]) for i, (c, _) in enumerate(items)])
        for c in cams:
            if c.ref_mode == "previous" and id(c) in want["last_ref"]:
                c.R = want["last_ref"][id(c)]
        assert np.array_equal(got["ssd"], want["ssd"]), b
        assert np.array_equal(got["sdd_pass"], want["sdd_pass"]), b
        assert np.array_equal(got["survivor_idx"], want["survivor_idx"]), b
        check_snm(got["logit"], got["snm_pass"], got["snm_class"], want["logit"], [cams[c] for c, _ in items],
                  want["survivors"])
        outs.append(got)
    for c in cams[:2]:
        assert np.array_equal(c.st.reference(), c.R)
    # the background-mode stream's reference never moves
    assert np.array_equal(cams[2].st.reference(), cams[2].R)
    passed = sum(int(o["sdd_pass"].sum()) for o in outs)
    assert 0 < passed < 30
    for c in cams:
        c.st.close()


def test_previous_frame_mode_prepared_batch_replays(env):
    """A prepared batch (CUDA graph) replayed three times over the same device frames: the first replay compares
    against the seeded reference, later replays against the batch's own last frame (the chained state), exactly
    as the oracle does when fed the same frames three times."""
    import torch
    ff, ctx, dev = env
    W, H = 1280, 720
    v = synth.Video(seed=61, width=W, height=H, period=10, on_len=3)
    cam = Cam(ctx, v, 0, dev, k_ref=4, delta=3.0, ref_mode="previous")
    ts = list(range(10))
    host = cam.host_frames(ts)
    d = _dev(host, dev)
    b = ctx.prepare([(cam.st, d[i], t) for i, t in enumerate(ts)])
    cs = torch.cuda.Stream(device=dev)
    for rep in range(3):
        b.launch(cs)
        got = b.fetch(cs)
        want = oracle_for([(cam, host[i]) for i in range(10)])
        cam.R = want["last_ref"][id(cam)]
        assert np.array_equal(got["ssd"], want["ssd"]), rep
        assert np.array_equal(got["sdd_pass"], want["sdd_pass"]), rep
        check_snm(got["logit"], got["snm_pass"], got["snm_class"], want["logit"], [cam] * 10, want["survivors"])
    assert np.array_equal(cam.st.reference(), cam.R)
    b.destroy()
    cam.st.close()


def test_previous_frame_mode_host_frames(env):
    """ffsva_filter_batch_host (frames staged through the device ring in 32-frame chunks) with a previous-mode
    stream spanning several chunks."""
    ff, ctx, dev = env
    W, H = 640, 360
    v = synth.Video(seed=71, width=W, height=H, period=25, on_len=5)
    cam = Cam(ctx, v, 0, dev, k_ref=4, delta=30000.0, ref_mode="previous", distance="sad")
    ts = list(range(70))
    host = cam.host_frames(ts)
    got = ctx.filter_batch([(cam.st, host[i], t) for i, t in enumerate(ts)], host=True)
    want = oracle_for([(cam, host[i]) for i in range(70)])
    assert np.array_equal(got["ssd"], want["ssd"])
    assert np.array_equal(got["sdd_pass"], want["sdd_pass"])
    assert np.array_equal(cam.st.reference(), want["last_ref"][id(cam)])
    cam.st.close()


def test_scheduler_rejects_previous_mode(env):
    import ctypes
    ff, ctx, dev = env
    from paper_conf_icpp_zhangcjzly18_b200 import ffsva as ffb
    W, H = 200, 120
    v = synth.Video(seed=81, width=W, height=H)
    cam = Cam(ctx, v, 0, dev, k_ref=2, ref_mode="previous")
    d = _dev(cam.host_frames([0]), dev)
    L = ffb.lib()
    h = ctypes.c_void_p()
    assert L.ffsva_sched_create(dev.index or 0, 8, 8, ctypes.byref(h)) == ffb.FFSVA_OK
    fr = (ffb.Frame * 1)(ffb.Frame(cam.st.handle, d[0].data_ptr(), 0))
    acc = (ctypes.c_uint8 * 1)()
    assert L.ffsva_sched_push(h, fr, 1, acc) == ffb.FFSVA_EINVAL
    assert L.ffsva_sched_destroy(h) == ffb.FFSVA_OK
    cam.st.close()


@pytest.mark.parametrize("metric", ["mse", "sad"])
def test_previous_frame_mode_large_grid_no_wrap(env, metric):
    """PREVIOUS mode on a 1000x1000 SDD grid (one CTA per frame in K2): a black frame after a white one gives
    SSD = 3e6 * 255^2 = 1.95e11 (MSE) or 3e6 * 255 (SAD), far beyond 32 bits — the distance must not wrap."""
    import torch
    ff, ctx, dev = env
    W = H = 1000
    st = ctx.open_stream(width=W, height=H, delta_diff=0.0, sdd=(1000, 1000), ref_mode="previous", distance=metric)
    white = np.full((H, 3 * W), 255, np.uint8)
    st.set_reference(torch.from_numpy(white[None]).to(dev))
    frames = torch.from_numpy(np.stack([np.zeros((H, 3 * W), np.uint8), white, white])).to(dev)
    got = ctx.sdd_batch([(st, frames[i], i) for i in range(3)], want_d100=False)
    n = 3 * W * H
    big = n * (255 * 255 if metric == "mse" else 255)
    assert [int(x) for x in got["ssd"]] == [big, big, 0]
    assert [int(x) for x in got["sdd_pass"]] == [1, 1, 0]
    st.close()
