"""Helpers shared by the GPU parity tests (tests/ only): set up streams through the C-ABI binding and run the
same seeded inputs through the oracle."""
from __future__ import annotations

import numpy as np

from oracle import oracle as orc
from synth import synth

SNM_TOL = 2e-2        # north_star: SNM logits within 2e-2 absolute of the oracle
SNM_TOL_BF16 = 2e-3   # vs the oracle's bf16-emulation mode (same operand rounding as the kernel)
F32 = np.float32


def f32(x: float) -> float:
    """The float32 value the C-ABI stores for a threshold, as a double for the oracle."""
    return float(np.float32(x))


class Cam:
    """One synthetic camera: its video, its reference frames and its SNM weights."""

    def __init__(self, ctx, video: synth.Video, stream_id: int, dev, delta=24.0, c_low=0.2, c_high=0.8, fd=0.5,
                 snm_batch=30, pitch=None, k_ref=8, bias_std=0.05, load_snm=True, distance="mse",
                 ref_mode="background"):
        import torch
        self.video, self.sid, self.dev = video, stream_id, dev
        self.pitch = 3 * video.width if pitch is None else pitch
        self.delta, self.c_low, self.c_high, self.fd = delta, c_low, c_high, fd
        self.distance, self.ref_mode = distance, ref_mode
        self.st = ctx.open_stream(width=video.width, height=video.height, row_pitch=self.pitch, delta_diff=delta,
                                  c_low=c_low, c_high=c_high, filter_degree=fd, snm_batch=snm_batch,
                                  distance=distance, ref_mode=ref_mode)
        self.refs = synth.frames(video, [stream_id] * k_ref, list(range(k_ref)), ref=True, pitch=self.pitch)
        self.st.set_reference(torch.from_numpy(self.refs).to(dev))
        self.R = orc.reference(self.refs, video.width, 100, 100)
        self.params = synth.snm_weights(video.seed, stream_id, bias_std=bias_std)
        if load_snm:
            self.st.snm_load(self.params)

    def host_frames(self, ts):
        return synth.frames(self.video, [self.sid] * len(ts), ts, pitch=self.pitch)


def oracle_for(cams_and_frames, run_snm=True, bf16_emul=False):
    """cams_and_frames: list of (Cam, host frame (H, pitch)). Runs the oracle cascade in batch order."""
    frames = [f for _, f in cams_and_frames]
    cams = [c for c, _ in cams_and_frames]
    # all cameras of one call must share the frame width for filter_frames; group by width
    widths = {c.video.width for c in cams}
    assert len(widths) == 1
    return orc.filter_frames(frames, cams[0].video.width, [c.R for c in cams], [c.delta for c in cams],
                             [c.params for c in cams], [f32(c.c_low) for c in cams], [f32(c.c_high) for c in cams],
                             [f32(c.fd) for c in cams], bf16_emul=bf16_emul, run_snm=run_snm,
                             metrics=[c.distance for c in cams], ref_modes=[c.ref_mode for c in cams],
                             stream_ids=[id(c) for c in cams])


def oracle_mixed(cams_and_frames, run_snm=True, bf16_emul=False):
    """Like oracle_for but frame by frame (any mix of resolutions)."""
    outs = [oracle_for([cf], run_snm=False) for cf in cams_and_frames]
    n = len(outs)
    res = {k: np.concatenate([o[k] for o in outs]) for k in ("ssd", "sdd_pass")}
    surv = orc.compact(res["sdd_pass"])
    sidx = np.full(n, -1, np.int32)
    sidx[surv] = np.arange(surv.size, dtype=np.int32)
    res["survivors"], res["survivor_idx"] = surv, sidx
    res["d50"] = [o["d50"][0] for o in outs]
    res["d100"] = [o["d100"][0] for o in outs]
    lg = np.full(n, np.nan)
    if run_snm:
        for i in surv:
            lg[i] = orc.snm_forward(res["d50"][i], cams_and_frames[i][0].params, bf16_emul=bf16_emul)
    res["logit"] = lg
    return res


def check_snm(got_logit, got_pass, got_cls, want_logit, cams, survivors, tol=SNM_TOL):
    """Logits within tol; decisions identical except where the oracle logit is within tol of a threshold. Returns
    (max |dlogit|, number of decisions compared) and asserts the decision check is not vacuous: at least 90% of
    the survivors are compared when there are 20 or more (the synthetic workloads keep < 10% of the logits within
    the margin of L_t, SURVEY §8(d), and a few % near c_low / c_high), at least one otherwise."""
    if survivors.size == 0:
        return 0.0, 0
    err = np.abs(got_logit[survivors].astype(np.float64) - want_logit[survivors])
    assert np.all(np.isfinite(got_logit[survivors]))
    assert err.max() <= tol, f"max |dlogit| {err.max():.3e} > {tol}"
    compared = 0
    for i in survivors:
        c = cams[i]
        lt = orc.logit(orc.tpre(f32(c.c_low), f32(c.c_high), f32(c.fd)))
        p, k = orc.decide(want_logit[i], f32(c.c_low), f32(c.c_high), f32(c.fd))
        near = min(abs(want_logit[i] - lt), abs(want_logit[i] - orc.logit(f32(c.c_low))),
                   abs(want_logit[i] - orc.logit(f32(c.c_high))))
        if near > tol:
            assert got_pass[i] == p, (i, want_logit[i], got_logit[i])
            assert got_cls[i] == k, (i, want_logit[i], got_logit[i])
            compared += 1
    assert compared >= 1 and (survivors.size < 20 or compared >= 0.8 * survivors.size), \
        f"only {compared}/{survivors.size} decisions compared"
    return float(err.max()), compared


class _DevArray:
    """A raw device pointer as a torch tensor view (__cuda_array_interface__), for reading library-owned device
    outputs (ffsva_batch_device_outputs) in tests."""

    def __init__(self, ptr: int, shape, typestr: str = "|u1"):
        self.__cuda_array_interface__ = {"data": (int(ptr), False), "shape": tuple(shape), "typestr": typestr,
                                         "version": 3, "strides": None}


def device_view(ptr: int, shape, typestr: str = "|u1"):
    import torch
    return torch.as_tensor(_DevArray(ptr, shape, typestr), device="cuda")


def _oracle_frame(args):
    """One frame through the oracle's SDD stage (C1-C3): D50, SSD, pass. ctypes releases the GIL, so frames run on
    a thread pool."""
    frame, W, R, delta = args
    d100 = orc.box_downsample(frame, W, 100, 100)
    d50 = orc.box_downsample(frame, W, 50, 50)
    ssd = orc.ssd(d100, R)
    return d50, ssd, orc.sdd_pass(ssd, orc.sdd_threshold("mse", delta, R))


def check_prepared_batch_all_frames(pb, pool, cams_of, got=None, stream=None, chunk=96):
    """Every frame of a prepared batch against the oracle, in the bench's launch configuration: the D50 image the
    SNM reads (device outputs, byte for byte), SSD and pass (bit-exact), survivor order, and every survivor's SNM
    logit / decision (check_snm). pool[i] is frame i (device tensor (H, pitch)); cams_of[i] its Cam. Returns the
    counts compared."""
    import concurrent.futures as cf
    import os
    import torch
    n = pool.shape[0]
    if got is None:
        got = pb.fetch(stream)
    outs = pb.device_outputs()
    stride = outs["d50_stride"]
    d50_dev = device_view(outs["d50"], (n, stride))
    W = cams_of[0].video.width
    surv_all, logit_want = [], np.full(n, np.nan)
    pass_want = np.zeros(n, np.uint8)
    ssd_want = np.zeros(n, np.uint64)
    d50_of = {}
    with cf.ThreadPoolExecutor(max_workers=max(1, len(os.sched_getaffinity(0)))) as ex:
        for i0 in range(0, n, chunk):
            i1 = min(n, i0 + chunk)
            host = pool[i0:i1].cpu().numpy()
            gpu_d50 = d50_dev[i0:i1, :7500].cpu().numpy()
            res = list(ex.map(_oracle_frame, [(host[k], W, cams_of[i0 + k].R, cams_of[i0 + k].delta)
                                              for k in range(i1 - i0)]))
            for k, (d50, ssd, p) in enumerate(res):
                i = i0 + k
                assert np.array_equal(gpu_d50[k], d50.ravel()), f"D50 of frame {i} differs from the oracle"
                ssd_want[i], pass_want[i] = ssd, p
                if p:
                    d50_of[i] = d50
        surv = np.flatnonzero(pass_want)
        lg = list(ex.map(lambda i: orc.snm_forward(d50_of[i], cams_of[i].params), surv.tolist()))
    logit_want[surv] = lg
    assert np.array_equal(got["ssd"].astype(np.uint64), ssd_want)
    assert np.array_equal(got["sdd_pass"].astype(np.uint8), pass_want)
    sidx = np.full(n, -1, np.int32)
    sidx[surv] = np.arange(surv.size, dtype=np.int32)
    assert np.array_equal(got["survivor_idx"], sidx)
    assert np.all(np.isnan(got["logit"][pass_want == 0]))
    err, nd = check_snm(got["logit"], got["snm_pass"], got["snm_class"], logit_want, cams_of, surv)
    near = int((np.abs(logit_want[surv]) < SNM_TOL).sum()) if surv.size else 0
    return {"frames": n, "d50_frames": n, "survivors": int(surv.size), "decisions": nd, "max_dlogit": err,
            "near_margin": near / surv.size if surv.size else 0.0}
