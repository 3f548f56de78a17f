"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times (prepared batch, replayed
as a CUDA graph on a side stream), EVERY frame against the oracle:

  M2    30 x 1280x720 streams, one second (30 frames) each (configs[1], the bench default)
  M3    offline 1920x1080, one stream, a batch of 512 frames (configs[2]); plus the whole hour: all 108,000 frames
        (frame t = pool[t mod 1500]) checked by lookup against the oracle's results for the 1,500 pool frames
  M4    64 x 1280x720 streams, one second (30 frames) each, TOR 1 / 10 / 50 % (configs[3])
  M5    256 x 1920x1080 streams, 10 frames each, one planted target per stream (configs[4], one GPU's shard at G=1)

Per frame (north_star): the 50x50 image the SNM reads (ffsva_batch_device_outputs, byte for
byte), the SSD and the pass flag (bit-exact), the stable survivor order (a4, Q16), every survivor's SNM logit
within 2e-2 with identical decisions outside that margin of a threshold (check_snm counts them), and every SDD
decision equal to the planted schedule (P8).
"""
import numpy as np
import pytest

from gpu_util import SNM_TOL, Cam, check_prepared_batch_all_frames, f32, oracle_for
from oracle import oracle as orc
from synth import synth

pytestmark = pytest.mark.gpu

# (streams, W, H, frames per stream in the batch, first frame, period, on_len, seed) — as bench.py CONFIGS
FULL = {
    "m2": (30, 1280, 720, 30, 120, 300, 30, 1002),
    "m3": (1, 1920, 1080, 512, 0, 300, 30, 1003),
    "m4_1": (64, 1280, 720, 30, 0, 300, 3, 1004),
    "m4_10": (64, 1280, 720, 30, 0, 300, 30, 1004),
    "m4_50": (64, 1280, 720, 30, 0, 300, 150, 1004),
    "m5": (256, 1920, 1080, 10, 0, 10, 1, 1005),
}


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


@pytest.mark.parametrize("name", list(FULL))
def test_full_size_config_every_frame(env, name):
    ff, ctx, dev = env
    import torch
    S, W, H, F, t0, period, on_len, seed = FULL[name]
    v = synth.Video(seed=seed, width=W, height=H, period=period, on_len=on_len)
    cams = [Cam(ctx, v, s, dev, k_ref=2, snm_batch=30) for s in range(S)]
    sid = torch.arange(S, dtype=torch.int32, device=dev).repeat_interleave(F)
    ts = (torch.arange(F, dtype=torch.int64, device=dev) + t0).repeat(S)
    pool = torch.empty((S * F, H, 3 * W), dtype=torch.uint8, device=dev)
    synth.frames_cuda(v, sid, ts, pool, H * 3 * W, 3 * W)
    torch.cuda.synchronize()
    items = [(cams[i // F].st, pool[i], t0 + i % F) for i in range(S * F)]
    pb = ctx.prepare(items)
    s = torch.cuda.Stream()
    pb.launch(s)
    pb.launch(s)  # graph replay: the second launch must give the same results
    got = pb.fetch(s)

    # full size: every decision equals the planted schedule; survivors in stable batch order
    sid_h, ts_h = sid.cpu().numpy(), ts.cpu().numpy()
    want_pass = np.array([int(synth.is_target(v, int(sid_h[i]), int(ts_h[i]))) for i in range(S * F)], np.uint8)
    assert np.array_equal(got["sdd_pass"].astype(np.uint8), want_pass)
    planted = sum(synth.planted(v, k, t0, t0 + F) for k in range(S))
    assert int(got["sdd_pass"].sum()) == planted
    surv = np.flatnonzero(want_pass)
    sidx = np.full(S * F, -1, np.int32)
    sidx[surv] = np.arange(surv.size, dtype=np.int32)
    assert np.array_equal(got["survivor_idx"], sidx)
    assert np.all(np.isnan(got["logit"][want_pass == 0]))
    assert np.all(np.isfinite(got["logit"][surv]))

    # every frame against the oracle (D50 the SNM reads, SSD, pass, order, all survivors' SNM)
    counts = check_prepared_batch_all_frames(pb, pool, [cams[i // F] for i in range(S * F)], got=got)
    assert counts["survivors"] == planted and counts["d50_frames"] == S * F
    assert counts["near_margin"] < 0.10, counts
    print(name, counts)
    pb.destroy()
    for c in cams:
        c.st.close()


def test_m3_whole_hour_by_lookup(env):
    """M3 (configs[2]): one 1080p stream for an hour, 108,000 frames, frame t = pool[t mod 1500].
    The oracle computes all 1,500 pool frames; the GPU runs all 108,000 frames in the bench's launch
    configuration (prepared batches of 512 replayed as CUDA graphs) and every result is checked by lookup:
    SSD and pass bit-exact, logits within 2e-2, decisions identical outside the margin, survivor ranks stable."""
    ff, ctx, dev = env
    import concurrent.futures as cf
    import os
    import torch
    W, H, PF, T, B = 1920, 1080, 1500, 108_000, 512
    v = synth.Video(seed=1003, width=W, height=H, period=300, on_len=30)
    cam = Cam(ctx, v, 0, dev, k_ref=2, snm_batch=30)
    pool = torch.empty((PF, H, 3 * W), dtype=torch.uint8, device=dev)
    synth.frames_cuda(v, torch.zeros(PF, dtype=torch.int32, device=dev), torch.arange(PF, dtype=torch.int64,
                      device=dev), pool, H * 3 * W, 3 * W)
    torch.cuda.synchronize()
    # oracle on the 1,500 pool frames (threads: ctypes releases the GIL)
    ssd_o = np.zeros(PF, np.uint64)
    pass_o = np.zeros(PF, np.uint8)
    logit_o = np.full(PF, np.nan)
    T_mse = orc.sdd_threshold("mse", 24.0, cam.R)

    def one(p):
        h = pool_h[p - p0]
        d100 = orc.box_downsample(h, W, 100, 100)
        s_ = orc.ssd(d100, cam.R)
        ps = orc.sdd_pass(s_, T_mse)
        lg = orc.snm_forward(orc.box_downsample(h, W, 50, 50), cam.params) if ps else np.nan
        return s_, ps, lg

    with cf.ThreadPoolExecutor(max_workers=max(1, len(os.sched_getaffinity(0)))) as ex:
        for p0 in range(0, PF, 100):
            pool_h = pool[p0:p0 + 100].cpu().numpy()
            for k, (s_, ps, lg) in enumerate(ex.map(one, range(p0, min(PF, p0 + 100)))):
                ssd_o[p0 + k], pass_o[p0 + k], logit_o[p0 + k] = s_, ps, lg
    assert int(pass_o.sum()) == synth.planted(v, 0, 0, PF)
    lt = orc.logit(orc.tpre(f32(0.2), f32(0.8), f32(0.5)))
    s = torch.cuda.Stream()
    checked = decisions = 0
    for b0 in range(0, T, B):
        ts = np.arange(b0, min(T, b0 + B))
        pb = ctx.prepare([(cam.st, pool[t % PF], int(t)) for t in ts])
        pb.launch(s)
        got = pb.fetch(s)
        p = ts % PF
        assert np.array_equal(got["ssd"].astype(np.uint64), ssd_o[p])
        assert np.array_equal(got["sdd_pass"].astype(np.uint8), pass_o[p])
        surv = np.flatnonzero(pass_o[p])
        sidx = np.full(ts.size, -1, np.int32)
        sidx[surv] = np.arange(surv.size, dtype=np.int32)
        assert np.array_equal(got["survivor_idx"], sidx)
        err = np.abs(got["logit"][surv].astype(np.float64) - logit_o[p[surv]])
        assert surv.size == 0 or err.max() <= SNM_TOL
        for j in surv:
            w = logit_o[p[j]]
            if min(abs(w - lt), abs(w - orc.logit(f32(0.2))), abs(w - orc.logit(f32(0.8)))) > SNM_TOL:
                wp, wc = orc.decide(w, f32(0.2), f32(0.8), f32(0.5))
                assert got["snm_pass"][j] == wp and got["snm_class"][j] == wc
                decisions += 1
        checked += ts.size
        pb.destroy()
    assert checked == T and decisions >= 0.8 * (T // PF) * int(pass_o.sum())
    cam.st.close()
