"""GPU test of the online runtime (§4.3): per-stream queues, feedback thresholds, dynamic batching.

Every accepted frame must come back exactly once with the same SDD result as the oracle (bit-exact) and an
SNM logit within tolerance; the feedback queue must actually engage (refused pushes, blocked SDD admissions)
and the queue depths must respect their thresholds at every cycle."""
import numpy as np
import pytest

from gpu_util import SNM_TOL, Cam, f32
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


@pytest.mark.parametrize("pipeline,W,H", [(False, 640, 360), (True, 640, 360), (False, 1280, 720),
                                          (True, 1280, 720)])
def test_online_feedback_queue_and_dynamic_batching(env, pipeline, W, H):
    """Synchronous and pipelined ticks (ffsva_sched_set_pipeline): same per-frame results, every frame once. The
    SNM's input in the online runtime is the device slot pool: after every tick, the image every admitted frame
    got (K1 -> its slot) and the image every popped frame is scored from (possibly written cycles earlier) are read
    back (ffsva_sched_inspect) and compared with the oracle's 50x50 resize byte for byte."""
    ff, ctx, dev = env
    import torch
    from paper_conf_icpp_zhangcjzly18_b200.ffsva import Scheduler
    q_sdd, q_snm, B = 2, 3, 1
    v = synth.Video(seed=61, width=W, height=H, period=10, on_len=5)
    cams = []
    for s in range(3):
        c = Cam(ctx, v, s, dev, k_ref=2, snm_batch=B)
        cams.append(c)
    # rebuild the streams with the online thresholds (Cam opens with the defaults)
    for c in cams:
        c.st.close()
        c.st = ctx.open_stream(width=W, height=H, delta_diff=24.0, snm_batch=B, q_sdd=q_sdd, q_snm=q_snm)
        c.st.set_reference(torch.from_numpy(c.refs).to(dev))
        c.st.snm_load(c.params)
    T = 24
    host = {s: c.host_frames(list(range(T))) for s, c in enumerate(cams)}
    dev_frames = {s: torch.from_numpy(host[s]).to(dev) for s in host}
    want_d50 = {(s, t): orc.box_downsample(host[s][t], W, 50, 50) for s in host for t in range(T)}
    at_ptr = {dev_frames[s][t].data_ptr(): (s, t) for s in host for t in range(T)}
    checked = {0: 0, 1: 0}
    sched = Scheduler(ctx, max_frames_per_tick=64, snm_slots=64)
    assert sched.set_pipeline(pipeline)
    ctx.stats(reset=True)
    # pipelined: a cycle's survivors join the SNM queue one tick later, after the next admission check
    snm_slack = 6 if pipeline else 3
    handle_to_s = {c.st.handle: s for s, c in enumerate(cams)}
    backlog = {s: list(range(T)) for s in range(3)}
    got = {}
    refused = blocked = 0
    cs = torch.cuda.Stream()
    for step in range(200):
        items = []
        for s in range(3):  # each prefetcher offers its next 3 frames; refused frames stay in its backlog
            for t in backlog[s][:3]:
                items.append((cams[s].st, dev_frames[s][t], t))
        if items:
            acc = sched.push(items)
            refused += int((acc == 0).sum())
            for (st, _, t), a in zip(items, acc):
                if a:
                    backlog[handle_to_s[st.handle]].remove(t)
        ev, info = sched.tick(cs)
        blocked += info["sdd_blocked"]
        cyc = sched.inspect()
        assert (cyc["stage"] == 0).sum() == info["admitted"] and (cyc["stage"] == 1).sum() == info["snm_scored"]
        for fr, stg, img in zip(cyc["frames"], cyc["stage"], cyc["d50"]):
            key = at_ptr[int(fr["pixels"])]
            assert int(fr["frame_no"]) == key[1]
            assert np.array_equal(img, want_d50[key]), ("slot-pool D50 differs", stg, key)
            checked[int(stg)] += 1
        for c in cams:
            d_sdd, d_snm = sched.depth(c.st)
            assert d_sdd <= q_sdd + 1, "SDD queue grew past its threshold + 1"
            assert d_snm <= q_snm + snm_slack, "SNM queue grew past threshold + the in-flight cycles' admissions"
        for e in ev:
            key = (handle_to_s[int(e["stream"])], int(e["frame_no"]))
            assert key not in got, "frame reported twice"
            got[key] = e["result"]
        if all(not b for b in backlog.values()) and info["sdd_queued"] == 0 and info["snm_queued"] == 0 \
                and info["events_pending"] == 0:
            break
    sched.destroy()
    assert len(got) == 3 * T, f"{len(got)} of {3 * T} frames reported"
    n_surv = sum(int(synth.is_target(v, s, t)) for s in range(3) for t in range(T))
    assert checked[0] == 3 * T and checked[1] == n_surv > 0, checked  # every admission, every pop
    # a8 statistics of the online runtime: kernel counters vs the oracle-derived schedule, and the latency
    # histogram (one entry per reported frame; push -> report within this test's wall time)
    st = ctx.stats()
    for s_, c in enumerate(cams):
        row = st[c.st.slot]
        assert row[0] == T and row[1] == sum(int(synth.is_target(v, s_, t)) for t in range(T))
        assert row[8] == T and int(row[10:24].sum()) == T, row
        assert 0 < row[9] <= T * 600e6
    assert refused > 0, "the SDD-queue threshold never refused a push"
    assert blocked > 0, "the SNM-queue threshold never blocked the SDD stage"
    for (s, t), r in got.items():
        c = cams[s]
        w = orc.filter_frames([host[s][t]], W, [c.R], [24.0], [c.params], [f32(0.2)], [f32(0.8)], [f32(0.5)])
        assert int(r["ssd"]) == int(w["ssd"][0]), (s, t)
        assert int(r["sdd_pass"]) == int(w["sdd_pass"][0]), (s, t)
        assert r["sdd_pass"] == int(synth.is_target(v, s, t))
        if w["sdd_pass"][0]:
            assert abs(float(r["logit"]) - w["logit"][0]) <= SNM_TOL, (s, t)
        else:
            assert np.isnan(r["logit"])


@pytest.mark.parametrize("policy", ["static", "feedback"])
def test_fixed_size_batch_policies(env, policy):
    """f4 (§4.3.2, §5.4): under STATIC every SNM pop is exactly BatchSize frames until the end of
    input is drained in DYNAMIC mode; under FEEDBACK a pop is either a full batch or a queue that blocked its SDD
    stage (> q_snm frames). Every frame still comes back once with the oracle's SDD result."""
    ff, ctx, dev = env
    import torch
    from paper_conf_icpp_zhangcjzly18_b200.ffsva import Scheduler
    B, q_snm = 4, 5
    v = synth.Video(seed=67, width=640, height=360, period=6, on_len=5)
    cams = [Cam(ctx, v, s, dev, k_ref=2, load_snm=True) for s in range(2)]
    for c in cams:
        c.st.close()
        c.st = ctx.open_stream(width=640, height=360, delta_diff=24.0, snm_batch=B, q_sdd=2, q_snm=q_snm)
        c.st.set_reference(torch.from_numpy(c.refs).to(dev))
        c.st.snm_load(c.params)
    T = 30
    dev_frames = [torch.from_numpy(c.host_frames(list(range(T)))).to(dev) for c in cams]
    sched = Scheduler(ctx, max_frames_per_tick=64, snm_slots=64)
    sched.set_policy(policy)
    nxt = [0, 0]
    got = {}
    cs = torch.cuda.Stream()
    for step in range(400):
        items = [(cams[s].st, dev_frames[s][t], t) for s in range(2) for t in range(nxt[s], min(T, nxt[s] + 3))]
        if items:
            acc = sched.push(items)
            for (st, _, t), a in zip(items, acc):
                s = 0 if st is cams[0].st else 1
                if a and t == nxt[s]:
                    nxt[s] += 1
        if nxt == [T, T]:
            sched.set_policy("dynamic")  # end of input: drain partial batches
        ev, info = sched.tick(cs)
        if nxt != [T, T] and info["snm_batches"]:
            if policy == "static":  # exactly BatchSize per pop
                assert info["snm_scored"] == B * info["snm_batches"], info
            else:  # each pop is BatchSize frames or a whole blocking queue (> q_snm >= B frames)
                assert info["snm_scored"] >= B * info["snm_batches"], info
        for e in ev:
            key = (0 if int(e["stream"]) == cams[0].st.handle else 1, int(e["frame_no"]))
            assert key not in got
            got[key] = e["result"]
        if nxt == [T, T] and info["sdd_queued"] == 0 and info["snm_queued"] == 0 and info["events_pending"] == 0:
            break
    sched.destroy()
    assert len(got) == 2 * T
    for (s, t), r in got.items():
        assert r["sdd_pass"] == int(synth.is_target(v, s, t)), (s, t)
    # every frame against the oracle: the batch trigger changes timing only, never a frame's result (C8)
    for s, c in enumerate(cams):
        host = c.host_frames(list(range(T)))
        w = orc.filter_frames(list(host), 640, [c.R] * T, [24.0] * T, [c.params] * T, [f32(0.2)] * T, [f32(0.8)] * T,
                              [f32(0.5)] * T)
        for t in range(T):
            r = got[(s, t)]
            assert int(r["ssd"]) == int(w["ssd"][t]) and int(r["sdd_pass"]) == int(w["sdd_pass"][t]), (s, t)
            if w["sdd_pass"][t]:
                assert abs(float(r["logit"]) - w["logit"][t]) <= SNM_TOL, (s, t)
    for c in cams:
        c.st.close()


@pytest.mark.parametrize("pipeline", [False, True])
def test_online_three_stage_cascade_with_tyolo(env, pipeline):
    """f1 in the online runtime (§3.1 Fig. 2): SDD -> SNM -> T-YOLO queue -> T-YOLO. Every frame comes back
    once; SNM survivors carry a T-YOLO count equal to the standalone stage's on the same frame and target class
    (one frame also against the fp64 oracle), tyolo_pass = count >= NumberofObjects (L195), everything else -1;
    the T-YOLO queue threshold (q_tyolo = 1) blocks the SNM stage (L209)."""
    ff, ctx, dev = env
    import torch
    from paper_conf_icpp_zhangcjzly18_b200.ffsva import Scheduler
    v = synth.Video(seed=71, width=640, height=360, period=4, on_len=3)
    params = synth.tyolo_weights(5, target_class=14)
    ty = ff.Tyolo(ctx, params)
    cams = [Cam(ctx, v, s, dev, k_ref=2) for s in range(2)]
    targets, noo = [14, 6], [2, 150]
    for s, c in enumerate(cams):  # reopen with the T-YOLO fields (c_low = 0: every SDD survivor passes the SNM)
        c.st.close()
        c.st = ctx.open_stream(width=640, height=360, delta_diff=24.0, c_low=0.0, c_high=0.0, filter_degree=0.0,
                               snm_batch=4, q_sdd=2, q_snm=4, number_of_objects=noo[s], target_class=targets[s],
                               q_tyolo=1)
        c.st.set_reference(torch.from_numpy(c.refs).to(dev))
        c.st.snm_load(c.params)
    T = 16
    host = {s: c.host_frames(list(range(T))) for s, c in enumerate(cams)}
    frames = {s: torch.from_numpy(host[s]).to(dev) for s in host}
    sched = Scheduler(ctx, max_frames_per_tick=64, snm_slots=64)
    sched.set_tyolo(ty, num_tyolo=1, thresh=0.2)
    assert sched.set_pipeline(pipeline)
    h2s = {c.st.handle: s for s, c in enumerate(cams)}
    nxt, got, snm_blocked, scored = [0, 0], {}, 0, 0
    for step in range(400):
        items = [(cams[s].st, frames[s][t], t) for s in range(2) for t in range(nxt[s], min(T, nxt[s] + 3))]
        if items:
            acc = sched.push(items)
            for (st, _, t), a in zip(items, acc):
                s = h2s[st.handle]
                if a and t == nxt[s]:
                    nxt[s] += 1
        ev, info = sched.tick()
        snm_blocked += info["snm_blocked"]
        scored += info["tyolo_scored"]
        for e in ev:
            key = (h2s[int(e["stream"])], int(e["frame_no"]))
            assert key not in got
            got[key] = e["result"]
        if nxt == [T, T] and info["sdd_queued"] == 0 and info["snm_queued"] == 0 and info["tyolo_queued"] == 0 \
                and info["events_pending"] == 0:
            break
    sched.set_tyolo(None)
    sched.destroy()
    assert len(got) == 2 * T
    assert snm_blocked > 0, "the T-YOLO queue threshold never blocked the SNM stage"
    reached = [(s, t) for (s, t), r in got.items() if r["snm_pass"]]
    assert scored == len(reached) > 0
    for (s, t), r in got.items():
        assert r["sdd_pass"] == int(synth.is_target(v, s, t))
        if r["snm_pass"]:
            assert r["tyolo_count"] >= 0 and r["tyolo_pass"] == int(r["tyolo_count"] >= noo[s])
        else:
            assert r["tyolo_count"] == -1 and r["tyolo_pass"] == 0
    for s in range(2):
        ts = [t for (ss, t) in reached if ss == s]
        if not ts:
            continue
        alone = ty.run([(cams[s].st, frames[s][t], t) for t in ts], target_class=targets[s], thresh=0.2)
        assert [int(got[(s, t)]["tyolo_count"]) for t in ts] == alone["counts"].tolist()
    s, t = reached[0]
    want = orc.tyolo_forward(orc.resize(host[s][t], 640, 416, 416), params, bf16_emul=True)
    sc = orc.tyolo_scores(want, targets[s])
    near = int((np.abs(sc - 0.2) <= 0.75 * 0.03).sum())  # the score margin of test_gpu_tyolo.py (TAU_HEAD)
    assert abs(int(got[(s, t)]["tyolo_count"]) - orc.tyolo_count(want, targets[s], 0.2)) <= near
    for c in cams:
        c.st.close()
    ty.destroy()
