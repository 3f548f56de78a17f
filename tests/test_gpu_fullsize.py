"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times (prepared batch, replayed
as a CUDA graph on a side stream), for the configs test_gpu_parity.py does not already cover at full size
(M2 is `test_full_size_config2_sampled` there):

  M3    offline 1920x1080, one stream, batches of 512 frames (configs[2])
  M4    64 x 1280x720 streams, one second (30 frames) each, TOR 1 / 10 / 50 % (configs[3])
  M5    256 x 1920x1080 streams, 10 frames each, one planted target per stream (configs[4], one GPU's shard at G=1)

Checked at full size: every frame's SDD decision equals the planted schedule
(so the pass count equals the planted count), survivor_idx is the stable rank among survivors (a4, Q16). Checked
element by element on sampled frames the oracle computes one by one: the SSD (bit-exact), and for sampled
survivors the SNM logit within 2e-2 with identical decisions outside that margin of a threshold (north_star).
"""
import numpy as np
import pytest

from gpu_util import SNM_TOL, Cam, check_snm, oracle_for
from synth import synth

pytestmark = pytest.mark.gpu

# (name, streams, W, H, frames per stream in the batch, first frame, period, on_len, seed) — as bench.py CONFIGS
FULL = {
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
def test_full_size_config_sampled(env, name):
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

    # sampled frames element by element against the oracle: non-survivors spread over the batch, the first and
    # last survivors, and survivors of the last stream (the batch's ragged tail of per-stream SNM pops)
    rng = np.random.default_rng(seed)
    non = np.flatnonzero(want_pass == 0)
    sample = sorted(set(rng.choice(non, size=min(10, non.size), replace=False).tolist()
                        + surv[:6].tolist() + surv[-4:].tolist()
                        + rng.choice(surv, size=min(6, surv.size), replace=False).tolist()))
    pairs = [(cams[i // F], cams[i // F].host_frames([int(ts_h[i])])[0]) for i in sample]
    w = oracle_for(pairs)
    idx = np.array(sample)
    assert np.array_equal(got["ssd"][idx].astype(np.uint64), w["ssd"].astype(np.uint64))
    assert np.array_equal(got["sdd_pass"][idx].astype(np.uint8), w["sdd_pass"].astype(np.uint8))
    ws_ = np.flatnonzero(w["sdd_pass"])
    check_snm(got["logit"][idx], got["snm_pass"][idx], got["snm_class"][idx], w["logit"], [p[0] for p in pairs],
              ws_, tol=SNM_TOL)
    pb.destroy()
    for c in cams:
        c.st.close()
