"""Paced online driver: S cameras at 30 FPS through the online runtime (ffsva_sched_*), for validating
"sustained 30-FPS streams": frame k of stream s becomes available at t0 + phi_s + k/30
(phi_s spreads the streams over one frame period); each cycle pushes every frame that has arrived (frames the
feedback queue refuses stay in the camera's backlog and are offered again next cycle), runs one scheduler tick
and records arrival->decision latency for every reported frame. A stream count is sustained when the p99
latency stays within the budget (the paper tolerates seconds) and no backlog accumulates.

The frames' bytes live in a device pool (the online measurement covers scheduling + kernels, not ingest I/O);
stream s replays content stream s % n_content with its own reference image and SNM."""
from __future__ import annotations

import time

import numpy as np


def sustained_verdict(arrivals_in_window: int, decided_in_window: int, p99_s: float, backlog_t, backlog_v, streams: int,
                      seconds: float, latency_budget_s: float = 1.0, min_decided: float = 0.99,
                      max_growth_per_stream_s: float = 0.05) -> dict:
    """A stream count is sustained when:
      * p99 arrival -> decision latency <= latency_budget_s (the paper tolerates seconds);
      * >= min_decided of the frames that arrived in the measurement window were decided by the end of the run;
      * the backlog (arrived, not yet decided frames) does not grow over the last min(10 s, half the run): the least-
        squares slope of backlog(t) is <= max_growth_per_stream_s frames per stream per second (0.05: less than half
        a frame per stream accumulated over 10 s).
    Host logic only (tested on CPU)."""
    t = np.asarray(backlog_t, dtype=np.float64)
    v = np.asarray(backlog_v, dtype=np.float64)
    tail = min(10.0, seconds / 2)
    m = t >= (t.max(initial=0.0) - tail) if t.size else np.zeros(0, bool)
    slope = float(np.polyfit(t[m], v[m], 1)[0]) if m.sum() >= 3 and np.ptp(t[m]) > 0 else 0.0
    frac = decided_in_window / arrivals_in_window if arrivals_in_window else 1.0
    ok = bool(p99_s <= latency_budget_s and frac >= min_decided and slope <= max_growth_per_stream_s * streams)
    return {"sustained": ok, "decided_fraction_of_window": frac, "backlog_slope_frames_per_s": slope,
            "backlog_slope_per_stream": slope / max(1, streams), "tail_seconds": tail,
            "criteria": f"p99 <= {latency_budget_s} s, decided >= {min_decided:.0%} of the window's arrivals, backlog "
                        f"slope over the last {tail:g} s <= {max_growth_per_stream_s} frames/stream/s"}


def run_paced(ctx, streams, content, n_content_frames, seconds, fps=30.0, tick_s=0.010, cuda_stream=None,
              latency_budget_s=1.0, tyolo=None, num_tyolo=4, pipelined=True, warmup_s=1.0):
    """streams[i]: ff.Stream; content[i]: (device frame tensor [n_content_frames, H, pitch]). tyolo: a Tyolo to run
    the full three-filter cascade (SDD -> SNM -> T-YOLO, f1) instead of SDD -> SNM. pipelined: ticks overlap the
    previous cycle's kernels with this driver's host work (ffsva_sched_set_pipeline). The measurement window is
    [warmup_s, seconds - latency_budget_s): frames arriving in it must be decided by the end of the run.

    Returns a dict of latency percentiles (driver clock: arrival = the camera's frame time; library: the a8
    histogram, arrival = accepted push), refusals, backlog trend, throughput and the sustained verdict."""
    import torch

    from .dist import summarize
    from .ffsva import FRAME_DTYPE, Scheduler

    S = len(streams)
    handles = np.array([s.handle for s in streams], dtype=np.uint64)
    order = np.argsort(handles)
    sorted_handles = handles[order]
    base_ptr = np.array([c.data_ptr() for c in content], dtype=np.uint64)
    fbytes = np.array([c[0].numel() for c in content], dtype=np.uint64)
    phase = (np.arange(S) * (1.0 / fps) / S).astype(np.float64)
    start_frame = (np.arange(S) * 37) % n_content_frames
    pushed = np.zeros(S, np.int64)          # frames handed to (and accepted by) the scheduler
    max_frames_tick = max(1024, int(S * fps * 0.25))
    sched = Scheduler(ctx, max_frames_per_tick=max_frames_tick, snm_slots=max(4096, S * 12))
    if tyolo is not None:
        sched.set_tyolo(tyolo, num_tyolo=num_tyolo)
    sched.set_pipeline(pipelined)
    slots = np.array([st.slot for st in streams], dtype=np.int64)
    ctx.stats(reset=True)  # the a8 latency histogram of this run only
    w0, w1 = warmup_s, max(warmup_s, seconds - latency_budget_s)
    ty_scored = 0
    lat, lat_win = [], []
    refused = 0
    done = 0
    decided_win = 0
    max_backlog = 0
    ticks = 0
    bt, bv = [], []  # backlog(t): arrived - decided frames over all streams
    tim = [0.0, 0.0, 0.0, 0.0, 0.0]  # python push, SDD cycle, SNM cycle, whole tick call, python events (s)
    try:
        torch.cuda.synchronize()
        t0 = time.perf_counter() + 0.05
        while True:
            now = time.perf_counter()
            el = now - t0
            if el > seconds:
                break
            due = np.floor((el - phase) * fps).astype(np.int64) + 1
            due = np.maximum(due, 0)
            want = due - pushed
            max_backlog = max(max_backlog, int(want.max(initial=0)))
            n_off = int(want.sum())
            if n_off > 0:
                # offer at most q_sdd + 1 frames per stream per cycle (the rest would be refused anyway)
                take = np.minimum(want, 3)
                idx = np.repeat(np.arange(S), take)
                k = pushed[idx] + (np.arange(idx.size) - np.repeat(np.cumsum(take) - take, take))
                fr = np.zeros(idx.size, dtype=FRAME_DTYPE)
                fr["stream"] = handles[idx]
                fr["pixels"] = base_ptr[idx] + ((start_frame[idx] + k) % n_content_frames).astype(np.uint64) * fbytes[idx]
                fr["frame_no"] = k
                acc = sched.push_array(fr)
                refused += int((acc == 0).sum())
                # accepted frames are a prefix per stream (a refusal stops the camera this cycle)
                pushed += np.bincount(idx[acc == 1], minlength=S)
            t_push = time.perf_counter()
            ev, info = sched.tick(cuda_stream)
            ticks += 1
            ty_scored += info["tyolo_scored"]
            t_done = time.perf_counter()
            tim[0] += t_push - now
            tim[1] += info["sdd_ms"] / 1e3
            tim[2] += info["snm_ms"] / 1e3
            tim[3] += t_done - t_push
            if ev.size:
                si = order[np.searchsorted(sorted_handles, ev["stream"])]
                arr = phase[si] + ev["frame_no"].astype(np.float64) / fps  # relative to t0
                L = t_done - (t0 + arr)
                lat.append(L)
                inw = (arr >= w0) & (arr < w1)
                lat_win.append(L[inw])
                decided_win += int(inw.sum())
                done += ev.size
            bt.append(t_done - t0)
            bv.append(float(np.maximum(due, 0).sum() - done))
            tim[4] += time.perf_counter() - t_done
            rest = tick_s - (time.perf_counter() - now)
            if rest > 0:
                time.sleep(rest)
        backlog_end = int((np.maximum(np.floor((time.perf_counter() - t0 - phase) * fps) + 1, 0) - pushed).sum())
    finally:
        sched.destroy()
    stats = ctx.stats(max_slots=int(slots.max()) + 1)
    lib = summarize(stats[slots]) if stats.shape[0] > slots.max() else {}
    # frames whose arrival lies in [w0, w1): stream s, frame k arrives at phase_s + k / fps
    arrivals_win = int((np.maximum(np.ceil((w1 - phase) * fps), 0) - np.maximum(np.ceil((w0 - phase) * fps), 0)).sum())
    L = np.concatenate(lat) if lat else np.zeros(1)
    Lw = np.concatenate(lat_win) if lat_win else np.zeros(1)
    if Lw.size == 0:
        Lw = np.zeros(1)
    p99 = float(np.percentile(Lw, 99))
    verdict = sustained_verdict(arrivals_win, decided_win, p99, bt, bv, S, seconds, latency_budget_s)
    res = {"streams": S, "seconds": seconds, "ticks": ticks, "frames_decided": int(done),
           "decided_fps": done / seconds, "offered_fps": S * fps, "refused_pushes": refused,
           "max_backlog_frames_per_stream": max_backlog, "backlog_frames_at_end": backlog_end,
           "window_s": [w0, w1], "arrivals_in_window": arrivals_win, "decided_in_window": decided_win,
           "latency_p50_s": float(np.percentile(Lw, 50)), "latency_p99_s": p99,
           "latency_max_s": float(L.max()),
           "library_latency": {k: lib[k] for k in ("decided", "latency_mean_ms", "latency_p50_ms_le",
                                                   "latency_p99_ms_le") if k in lib},
           "mean_ms_per_tick": {"push_py": 1e3 * tim[0] / max(1, ticks), "sdd_cycle": 1e3 * tim[1] / max(1, ticks),
                                "snm_cycle": 1e3 * tim[2] / max(1, ticks), "tick_call": 1e3 * tim[3] / max(1, ticks),
                                "events_py": 1e3 * tim[4] / max(1, ticks)}}
    res["pipelined"] = bool(pipelined)
    if tyolo is not None:
        res["stages"] = "SDD -> SNM -> T-YOLO (f1)"
        res["tyolo_scored"] = int(ty_scored)
    res.update(verdict)
    return res


def run_unpaced(ctx, streams, content, n_content_frames, seconds, policy="dynamic", cuda_stream=None,
                max_frames_per_tick=None, snm_slots=None):
    """Saturated run of the online runtime for the batch-mechanism comparison (§5.4, f4): every camera
    always has its next frame ready (the prefetcher re-offers whatever the feedback queue refused), so the
    decided-frame rate is the runtime's throughput; latency is push-acceptance -> decision of each frame.
    `policy` is the SNM batch trigger ('dynamic', 'feedback', 'static'; ffsva_sched_set_policy). After the timed
    window the policy switches to dynamic and the queues are drained (not counted)."""
    import torch

    from .ffsva import FRAME_DTYPE, Scheduler

    S = len(streams)
    handles = np.array([s.handle for s in streams], dtype=np.uint64)
    order = np.argsort(handles)
    sorted_handles = handles[order]
    base_ptr = np.array([c.data_ptr() for c in content], dtype=np.uint64)
    fbytes = np.array([c[0].numel() for c in content], dtype=np.uint64)
    start_frame = (np.arange(S) * 37) % n_content_frames
    q_sdd = np.array([s.desc.q_sdd for s in streams], dtype=np.int64)
    pushed = np.zeros(S, np.int64)
    RING = 1 << 14
    t_push = np.zeros((S, RING), np.float64)  # acceptance time of frame k of stream s at [s, k % RING]
    mf = max_frames_per_tick or max(256, S * 8)
    slots = snm_slots or max(1024, S * (max(s.desc.snm_batch for s in streams) + 16))
    sched = Scheduler(ctx, max_frames_per_tick=mf, snm_slots=slots)
    sched.set_policy(policy)
    lat, done, ticks, pops, scored = [], 0, 0, 0, 0
    try:
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        while True:
            now = time.perf_counter()
            if now - t0 > seconds:
                break
            take = q_sdd + 1
            idx = np.repeat(np.arange(S), take)
            k = pushed[idx] + (np.arange(idx.size) - np.repeat(np.cumsum(take) - take, take))
            fr = np.zeros(idx.size, dtype=FRAME_DTYPE)
            fr["stream"] = handles[idx]
            fr["pixels"] = base_ptr[idx] + ((start_frame[idx] + k) % n_content_frames).astype(np.uint64) * fbytes[idx]
            fr["frame_no"] = k
            acc = sched.push_array(fr) == 1
            t_push[idx[acc], k[acc] % RING] = time.perf_counter()
            pushed += np.bincount(idx[acc], minlength=S)
            ev, info = sched.tick(cuda_stream)
            t_done = time.perf_counter()
            ticks += 1
            pops += info["snm_batches"]
            scored += info["snm_scored"]
            if ev.size:
                si = order[np.searchsorted(sorted_handles, ev["stream"])]
                lat.append(t_done - t_push[si, ev["frame_no"] % RING])
                done += ev.size
        elapsed = time.perf_counter() - t0
        sched.set_policy("dynamic")
        for _ in range(10000):
            ev, info = sched.tick(cuda_stream)
            if info["sdd_queued"] == 0 and info["snm_queued"] == 0 and info["events_pending"] == 0:
                break
    finally:
        sched.destroy()
    L = np.concatenate(lat) if lat else np.zeros(1)
    return {"policy": policy, "streams": S, "seconds": elapsed, "ticks": ticks, "frames_decided": int(done),
            "fps": done / elapsed, "latency_mean_ms": 1e3 * float(L.mean()),
            "latency_p50_ms": 1e3 * float(np.percentile(L, 50)), "latency_p99_ms": 1e3 * float(np.percentile(L, 99)),
            "snm_scored": int(scored), "snm_batches": int(pops),
            "mean_snm_batch": scored / pops if pops else 0.0}



def run_controlled(ctx, owned, content, n_content_frames, n_cameras, seconds, spare_fps, interval_s=1.0,
                   window_s=2.0, stage="sdd", fps=30.0, tick_s=0.010, cuda_stream=None, device=None, max_streams=64,
                   q_snm_slots=4096):
    """Paced cameras through one instance's online runtime with the f2 controller in the loop (
    dist.Reforwarder). Every rank calls this at the same time with its own cameras (`owned`: global camera id ->
    Stream; cameras 0..n_cameras-1 in all) and the content of every camera (`content[gid]`: device frames
    [n_content_frames, H, pitch]) so a camera can continue wherever it is re-forwarded. Once per interval every rank
    reports its measured stage rate and per-stream overload, the plan is computed identically everywhere and moves
    are executed: the source stops its camera, ticks until the stream detaches, exports it; the target imports it
    and continues the camera at the frame the source had reached. `fps` is one rate for every camera or a dict gid ->
    frames/s. Returns this rank's decided frames per camera ({gid: {frame_no: result}}), the controller history and
    the cameras it owns at the end."""
    import torch

    from .dist import Reforwarder
    from .ffsva import FRAME_DTYPE, Scheduler

    rate = {g: float(fps[g] if isinstance(fps, dict) else fps) for g in range(n_cameras)}
    phase = {g: g * (1.0 / rate[g]) / max(1, n_cameras) for g in range(n_cameras)}
    sched = Scheduler(ctx, max_frames_per_tick=max(256, 8 * n_cameras), snm_slots=q_snm_slots)
    # images travel as device tensors whenever the process group is NCCL (dist._p2p_device), host tensors over gloo
    dev = device if device is not None else torch.device("cuda", ctx.device)
    rf = Reforwarder(ctx, sched, owned, spare_fps, window_s=window_s, stage=stage, device=dev)
    next_frame = {g: 0 for g in owned}
    decided = {}
    by_handle = {}

    def record(ev):
        for e in ev:
            g = by_handle[int(e["stream"])]
            decided.setdefault(g, {})[int(e["frame_no"])] = e["result"].copy()

    def drain(gid, st):  # the source side of a move: tick until the stream has left the scheduler
        for _ in range(10000):
            if sched.detach(st):
                return
            ev, _ = sched.tick(cuda_stream)
            record(ev)
        raise RuntimeError(f"camera {gid} never detached")

    n_steps = int(round(seconds / interval_s))
    steps = 0
    try:
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        while steps < n_steps:
            now = time.perf_counter()
            el = now - t0
            by_handle = {st.handle: g for g, st in owned.items()} | by_handle
            items = []
            for g, st in owned.items():
                due = int(np.floor((el - phase[g]) * rate[g])) + 1
                for k in range(next_frame[g], min(due, next_frame[g] + 3)):
                    items.append((g, st, k))
            if items:
                fr = np.zeros(len(items), dtype=FRAME_DTYPE)
                fr["stream"] = [st.handle for _, st, _ in items]
                fr["pixels"] = [content[g][k % n_content_frames].data_ptr() for g, _, k in items]
                fr["frame_no"] = [k for _, _, k in items]
                acc = sched.push_array(fr)
                for (g, _, k), a in zip(items, acc):
                    if a and k == next_frame[g]:
                        next_frame[g] = k + 1
            ev, info = sched.tick(cuda_stream)
            record(ev)
            rf.on_tick(time.perf_counter() - t0, info)
            if time.perf_counter() - t0 >= (steps + 1) * interval_s:
                rf.step(time.perf_counter() - t0, interval_s, max_streams, detach=drain, next_frame=next_frame)
                steps += 1
                by_handle = {st.handle: g for g, st in owned.items()} | by_handle
            rest = tick_s - (time.perf_counter() - now)
            if rest > 0:
                time.sleep(rest)
        for _ in range(1000):  # drain what is still queued
            ev, info = sched.tick(cuda_stream)
            record(ev)
            if info["sdd_queued"] == 0 and info["snm_queued"] == 0 and info["tyolo_queued"] == 0 and \
                    info["events_pending"] == 0:
                break
    finally:
        sched.destroy()
    return {"decided": decided, "history": rf.history, "owned": sorted(owned)}
