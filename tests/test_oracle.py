"""Pins of the CPU oracle against what the paper and the mathematics fix.

None of these re-types the oracle's own formula: each expected value is a hand-computed golden fixture
(tests/golden/, cited), a closed form, an invariant, brute force on a tiny input, or a library routine
(torch fp64 conv2d / max_pool2d) the definition reduces to.
"""
import json
import math
import os

import numpy as np
import pytest

from oracle import oracle as orc
from synth import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def _frame_from_channel0(ch0):
    a = np.asarray(ch0, dtype=np.uint8)
    H, W = a.shape
    f = np.zeros((H, W, 3), np.uint8)
    f[:, :, 0] = a
    return f.reshape(H, 3 * W), W


# ------------------------------------------------------------------ C1 downsample

def test_p3_hand_example_round_half_up():
    g = _gold("p3_downsample_4x4.json")
    f, W = _frame_from_channel0(g["channel0"])
    d = orc.box_downsample(f, W, *g["grid"])
    assert d[:, :, 0].tolist() == g["expected_d_channel0"]
    assert (d[:, :, 1:] == 0).all()
    s = orc.ssd(d, np.zeros_like(d))
    assert s == g["expected_ssd_vs_zero"]
    assert s != g["ssd_if_round_half_even"] and s != g["ssd_if_truncation"]


def test_p4_uneven_boxes():
    g = _gold("p4_downsample_5x3.json")
    f, W = _frame_from_channel0(g["channel0"])
    d = orc.box_downsample(f, W, *g["grid"])
    assert d[:, :, 0].tolist() == g["expected_d_channel0"]


@pytest.mark.parametrize("W,H,dw,dh", [(640, 360, 100, 100), (600, 400, 100, 100), (101, 103, 50, 50),
                                       (1280, 720, 50, 50), (100, 100, 100, 100), (7, 5, 3, 2)])
@pytest.mark.parametrize("v", [0, 1, 128, 254, 255])
def test_p2_constant_frame(W, H, dw, dh, v):
    f = np.full((H, 3 * W), v, np.uint8)
    d = orc.box_downsample(f, W, dw, dh)
    assert (d == v).all()


def test_p5_identity_grid():
    rng = np.random.default_rng(5)
    for W, H in [(100, 100), (13, 7), (1, 1)]:
        f = rng.integers(0, 256, size=(H, 3 * W), dtype=np.uint8)
        d = orc.box_downsample(f, W, W, H)
        assert np.array_equal(d.reshape(H, 3 * W), f)


def _brute_downsample(f, W, dw, dh):
    """Brute force from the interval definition via numpy slicing + exact integer rounding."""
    H = f.shape[0]
    img = f[:, :3 * W].reshape(H, W, 3).astype(np.int64)
    out = np.zeros((dh, dw, 3), np.int64)
    for oy in range(dh):
        ys = slice(oy * H // dh, (oy + 1) * H // dh)
        for ox in range(dw):
            xs = slice(ox * W // dw, (ox + 1) * W // dw)
            box = img[ys, xs]
            n = box.shape[0] * box.shape[1]
            s = box.sum(axis=(0, 1))
            # round half up = floor(s/n + 1/2), evaluated with Python fractions-free integer arithmetic
            out[oy, ox] = (2 * s + n) // (2 * n)
    return out.astype(np.uint8)


@pytest.mark.parametrize("W,H,dw,dh,pitch", [(37, 23, 10, 6, 37 * 3), (64, 36, 10, 10, 208), (23, 17, 23, 17, 69),
                                             (50, 40, 25, 20, 160)])
def test_downsample_brute_force(W, H, dw, dh, pitch):
    rng = np.random.default_rng(W * H)
    f = rng.integers(0, 256, size=(H, pitch), dtype=np.uint8)
    assert np.array_equal(orc.box_downsample(f, W, dw, dh), _brute_downsample(f, W, dw, dh))


def test_d50_is_union_of_d100_cells():
    """C1: floor(j*S/50) == floor(2j*S/100), so every 50-cell is exactly 2x2 100-cells (used by the kernel)."""
    for S in [100, 101, 360, 400, 600, 640, 720, 1080, 1280, 1920, 2160, 3840]:
        for j in range(51):
            assert (j * S) // 50 == (2 * j * S) // 100


# ------------------------------------------------------------------ C2 reference

def test_p1_reference_k1_is_downsample_and_ssd_zero():
    v = synth.Video(seed=3, width=640, height=360)
    f = synth.frame(v, 0, 0)
    r = orc.reference(f[None], 640, 100, 100)
    d = orc.box_downsample(f, 640, 100, 100)
    assert np.array_equal(r, d)
    s = orc.ssd(d, r)
    assert s == 0
    for delta in [0.0, 1e-9, 24.0]:
        assert orc.sdd_pass(s, orc.threshold(delta, 30000)) == 0


def test_reference_constant_frames_single_rounding():
    """K frames of constant value v_k: R = round_half_up(mean v_k) (one rounding, not a mean of rounded means)."""
    vals = [10, 11, 11, 12]  # mean 11.0
    fr = np.stack([np.full((9, 27), v, np.uint8) for v in vals])
    assert (orc.reference(fr, 9, 3, 3) == 11).all()
    vals = [0, 1]  # mean 0.5 -> half up -> 1
    fr = np.stack([np.full((4, 12), v, np.uint8) for v in vals])
    assert (orc.reference(fr, 4, 2, 2) == 1).all()
    vals = [0, 0, 1]  # mean 1/3 -> 0
    fr = np.stack([np.full((4, 12), v, np.uint8) for v in vals])
    assert (orc.reference(fr, 4, 2, 2) == 0).all()


def test_reference_brute_force():
    rng = np.random.default_rng(11)
    K, W, H = 5, 31, 19
    fr = rng.integers(0, 256, size=(K, H, 3 * W), dtype=np.uint8)
    got = orc.reference(fr, W, 7, 4)
    img = fr.reshape(K, H, W, 3).astype(np.int64)
    for oy in range(4):
        for ox in range(7):
            box = img[:, oy * H // 4:(oy + 1) * H // 4, ox * W // 7:(ox + 1) * W // 7]
            n = box.shape[0] * box.shape[1] * box.shape[2]
            s = box.sum(axis=(0, 1, 2))
            assert (got[oy, ox] == (2 * s + n) // (2 * n)).all()


# ------------------------------------------------------------------ C3 SSD / threshold

def test_ssd_closed_forms():
    a = np.full(30000, 255, np.uint8)
    b = np.zeros(30000, np.uint8)
    assert orc.ssd(a, b) == 30000 * 65025 == 1_950_750_000
    assert orc.ssd(b, a) == 1_950_750_000
    assert orc.ssd(a, a) == 0
    rng = np.random.default_rng(1)
    x = rng.integers(0, 256, 30000, dtype=np.uint8)
    y = rng.integers(0, 256, 30000, dtype=np.uint8)
    assert orc.ssd(x, y) == int(((x.astype(np.int64) - y.astype(np.int64)) ** 2).sum())


def test_threshold_strict_mse_greater_than_delta():
    """L151 'MSE larger than delta': exact boundary at SSD == floor(delta*N)."""
    N = 30000
    T = orc.threshold(24.0, N)
    assert T == 720000
    assert orc.sdd_pass(T, T) == 0 and orc.sdd_pass(T + 1, T) == 1
    # MSE > delta  <=>  SSD > T, checked with exact rationals over a sweep of fractional deltas
    from fractions import Fraction
    for delta in [0.0, 0.1, 1 / 3, 2.5, 24.000001, 100.7]:
        T = orc.threshold(delta, N)
        for s in [T - 1, T, T + 1]:
            if s < 0:
                continue
            assert orc.sdd_pass(s, T) == int(Fraction(s, N) > Fraction(delta))


# ------------------------------------------------------------------ C4 compaction (P9)

def test_p9_compaction_brute_force():
    rng = np.random.default_rng(2)
    for n in [0, 1, 7, 1000, 4097]:
        for p in [0.0, 0.1, 0.5, 1.0]:
            mask = (rng.random(n) < p).astype(np.uint8)
            got = orc.compact(mask)
            assert got.tolist() == [i for i in range(n) if mask[i]]


# ------------------------------------------------------------------ P8 planted count on synthetic video

@pytest.mark.parametrize("W,H,P,L", [(640, 360, 300, 30), (200, 120, 20, 5), (128, 104, 10, 1)])
def test_p8_sdd_pass_count_equals_planted(W, H, P, L):
    v = synth.Video(seed=1001, width=W, height=H, period=P, on_len=L)
    T = orc.threshold(24.0, 30000)
    n_frames = min(P, 60) if W >= 640 else P
    for s in range(2):
        refs = synth.frames(v, [s] * 32, list(range(32)), ref=True)
        R = orc.reference(refs, W, 100, 100)
        passed = 0
        for t in range(n_frames):
            f = synth.frame(v, s, t)
            p = orc.sdd_pass(orc.ssd(orc.box_downsample(f, W, 100, 100), R), T)
            assert p == int(synth.is_target(v, s, t)), (s, t)
            passed += p
        assert passed == synth.planted(v, s, 0, n_frames)


# ------------------------------------------------------------------ C6 conv / SNM

def test_p6_p7_conv_closed_forms():
    g = _gold("p6_p7_conv.json")
    imp = np.zeros((1, 3, 3))
    imp[0, 1, 1] = 1.0
    w = np.asarray(g["impulse_kernel"], np.float64)[None, None]
    assert orc.conv3x3(imp, w)[0].tolist() == g["impulse_expected"]
    ones = np.ones((1, 3, 3))
    assert orc.conv3x3(ones, np.ones((1, 1, 3, 3)))[0].tolist() == g["ones_expected"]


def test_maxpool_floor():
    x = np.arange(2 * 5 * 5, dtype=np.float64).reshape(2, 5, 5)
    p = orc.maxpool2(x)
    assert p.shape == (2, 2, 2)
    assert p[0].tolist() == [[6, 8], [16, 18]]


def _torch_snm(d50, params, c1, c2, bf16=False):
    """The same network through torch's fp64 library conv2d / max_pool2d / linear (library cross-check)."""
    import torch
    import torch.nn.functional as F
    h, w, _ = d50.shape
    p = torch.from_numpy(params.astype(np.float64))
    o = 0
    w1 = p[o:o + 27 * c1].view(c1, 3, 3, 3); o += 27 * c1
    b1 = p[o:o + c1]; o += c1
    w2 = p[o:o + 9 * c1 * c2].view(c2, c1, 3, 3); o += 9 * c1 * c2
    b2 = p[o:o + c2]; o += c2
    nf = c2 * (h // 2 // 2) * (w // 2 // 2)
    wfc = p[o:o + nf]; o += nf
    bfc = p[o]
    x = (torch.from_numpy(d50.astype(np.float64)).permute(2, 0, 1)[None] - 128.0) / 128.0
    a = F.max_pool2d(F.relu(F.conv2d(x, w1, b1, padding=1)), 2)
    if bf16:
        a = a.to(torch.bfloat16).to(torch.float64)
    a = F.max_pool2d(F.relu(F.conv2d(a, w2, b2, padding=1)), 2)
    return float(a.flatten() @ wfc + bfc)


@pytest.mark.parametrize("h,w,c1,c2", [(4, 4, 2, 2), (6, 5, 3, 2), (50, 50, 16, 32), (9, 11, 4, 8)])
def test_p11_snm_vs_torch_fp64(h, w, c1, c2):
    rng = np.random.default_rng(h * w + c1)
    d50 = rng.integers(0, 256, size=(h, w, 3), dtype=np.uint8)
    n = orc.snm_n_params(h, w, c1, c2)
    params = rng.normal(0, 0.5, n).astype(np.float32)
    got = orc.snm_forward(d50, params, c1, c2)
    want = _torch_snm(d50, params, c1, c2)
    assert abs(got - want) <= 1e-9 * max(1.0, abs(want))


def test_p11_bf16_emulation_vs_torch():
    """bf16 mode == torch with bf16-rounded weights and a bf16 cast of the pooled conv1 output."""
    import torch
    rng = np.random.default_rng(9)
    d50 = rng.integers(0, 256, size=(50, 50, 3), dtype=np.uint8)
    params = rng.normal(0, 0.2, orc.snm_n_params()).astype(np.float32)
    # round weights (not biases) to bf16 with torch (library RNE)
    pw = params.copy()
    c1, c2 = 16, 32
    nf = 4608
    segs = [(0, 27 * c1), (27 * c1 + c1, 27 * c1 + c1 + 9 * c1 * c2),
            (27 * c1 + c1 + 9 * c1 * c2 + c2, 27 * c1 + c1 + 9 * c1 * c2 + c2 + nf)]
    for a, b in segs:
        pw[a:b] = torch.from_numpy(params[a:b]).to(torch.bfloat16).float().numpy()
    got = orc.snm_forward(d50, params, bf16_emul=True)
    want = _torch_snm(d50, pw, c1, c2, bf16=True)
    assert abs(got - want) <= 1e-9 * max(1.0, abs(want))


def test_p10_snm_zero_weight_closed_forms():
    rng = np.random.default_rng(4)
    d50 = rng.integers(0, 256, size=(50, 50, 3), dtype=np.uint8)
    n = orc.snm_n_params()
    p = np.zeros(n, np.float32)
    p[-1] = 0.75
    assert orc.snm_forward(d50, p) == 0.75
    # w2 = 0, wfc = 1: logit = bfc + 144 * sum_k ReLU(b2_k)
    c1, c2 = 16, 32
    p = rng.normal(0, 1, n).astype(np.float32)
    o_w2 = 27 * c1 + c1
    o_b2 = o_w2 + 9 * c1 * c2
    p[o_w2:o_b2] = 0
    b2 = p[o_b2:o_b2 + c2]
    p[o_b2 + c2:-1] = 1.0
    want = float(p[-1]) + 144.0 * float(np.maximum(b2.astype(np.float64), 0).sum())
    assert abs(orc.snm_forward(d50, p) - want) < 1e-9


def test_round_bf16_against_torch():
    import torch
    rng = np.random.default_rng(6)
    xs = np.concatenate([rng.normal(0, 3, 5000), [1.0, 1 + 2 ** -8, 1 + 3 * 2 ** -8, -1 - 2 ** -8, 0.0, 2 ** -20,
                                                  65280.0, 1e10]]).astype(np.float32)
    want = torch.from_numpy(xs).to(torch.bfloat16).double().numpy()
    got = np.array([orc.round_bf16(float(x)) for x in xs])
    assert np.array_equal(got, want)
    assert orc.round_bf16(1 + 2 ** -8) == 1.0           # tie -> even
    assert orc.round_bf16(1 + 3 * 2 ** -8) == 1 + 2 ** -6


def test_generator_weights_are_bf16_exact():
    import torch
    p = synth.snm_weights(1, 0, bias_std=0.1)
    assert p.size == orc.snm_n_params() == 9697
    assert np.array_equal(torch.from_numpy(p).to(torch.bfloat16).float().numpy(), p)


# ------------------------------------------------------------------ C7 decision (P12)

def test_p12_eq2_and_logit_threshold():
    g = _gold("p12_eq2.json")
    for c in g["cases"]:
        t = orc.tpre(c["c_low"], c["c_high"], c["fd"])
        assert abs(t - c["t_pre"]) < 1e-15
        assert abs(orc.logit(t) - c["logit_threshold"]) < 1e-12


def test_decision_boundaries():
    # t_pre = 0.5 <=> logit >= 0 passes (c >= t_pre, L165)
    assert orc.decide(0.0, 0.2, 0.8, 0.5) == (1, 1)
    assert orc.decide(-1e-12, 0.2, 0.8, 0.5)[0] == 0
    # classes (L159): c < c_low -> 0, c > c_high -> 2, else 1
    assert orc.decide(math.log(0.1 / 0.9), 0.2, 0.8, 0.5) == (0, 0)
    assert orc.decide(math.log(0.9 / 0.1), 0.2, 0.8, 0.5) == (1, 2)
    # FilterDegree extremes: t_pre = c_low / c_high
    assert orc.decide(math.log(0.25 / 0.75), 0.2, 0.8, 0.0)[0] == 1
    assert orc.decide(math.log(0.25 / 0.75), 0.2, 0.8, 1.0)[0] == 0
    # t_pre = 0 -> everything passes; t_pre = 1 -> nothing passes
    assert orc.decide(-1e30, 0.0, 1.0, 0.0)[0] == 1
    assert orc.decide(1e30, 0.0, 1.0, 1.0)[0] == 0


# ------------------------------------------------------------------ f3 SDD variants: SAD, NRMSE (P13), previous-frame reference

def _d_from_channel0(ch0):
    a = np.asarray(ch0, dtype=np.uint8)
    d = np.zeros(a.shape + (3,), np.uint8)
    d[:, :, 0] = a
    return d


def test_p13_sad_hand_example():
    g = _gold("p13_sad_nrmse.json")
    d = _d_from_channel0(g["d_channel0"])
    assert orc.sad(d, np.zeros_like(d)) == g["expected_sad_vs_zero"]
    assert orc.sad(np.zeros_like(d), d) == g["expected_sad_vs_zero"]
    assert orc.sum_sq(d) == g["expected_sum_sq"]


def test_sad_invariants():
    """Invariants SAD must satisfy whatever its implementation: symmetry, triangle inequality, SAD == SSD when
    every |a - b| <= 1, and SSD <= SAD^2 <= N * SSD (Cauchy-Schwarz); closed form 255 * N."""
    rng = np.random.default_rng(13)
    N = 3000
    assert orc.sad(np.full(N, 255, np.uint8), np.zeros(N, np.uint8)) == 255 * N
    for _ in range(20):
        a, b, c = (rng.integers(0, 256, N, dtype=np.uint8) for _ in range(3))
        s_ab, s_bc, s_ac = orc.sad(a, b), orc.sad(b, c), orc.sad(a, c)
        assert s_ab == orc.sad(b, a)
        assert s_ac <= s_ab + s_bc
        q = orc.ssd(a, b)
        assert q <= s_ab * s_ab <= N * q
        e = np.clip(a.astype(np.int64) + rng.integers(-1, 2, N), 0, 255).astype(np.uint8)
        assert orc.sad(a, e) == orc.ssd(a, e)


def test_p13_nrmse_exact_boundary():
    """NRMSE(0, R=D) = 1 exactly (hand value): 'larger than' is strict, so delta = 1 drops the frame and the
    next double below 1 keeps it; 2D vs D gives the hand SSD 58."""
    g = _gold("p13_sad_nrmse.json")
    d = _d_from_channel0(g["d_channel0"])
    z = np.zeros_like(d)
    Q = orc.sum_sq(d)
    s = orc.ssd(z, d)
    assert s == Q == g["expected_sum_sq"]
    assert orc.sdd_pass(s, orc.sdd_threshold("nrmse", 1.0, d)) == 0
    assert orc.sdd_pass(s, orc.sdd_threshold("nrmse", math.nextafter(1.0, 0.0), d)) == 1
    d2 = np.clip(2 * d.astype(np.int64), 0, 255).astype(np.uint8)
    s2 = orc.ssd(d2, d)
    assert s2 == g["expected_ssd_2d_vs_d"]
    r = math.sqrt(s2 / Q)
    assert orc.sdd_pass(s2, orc.sdd_threshold("nrmse", r * (1 - 1e-12), d)) == 1
    assert orc.sdd_pass(s2, orc.sdd_threshold("nrmse", r * (1 + 1e-12), d)) == 0


def test_nrmse_threshold_against_float_definition():
    """Away from the boundary the exact test agrees with sqrt(SSD / sum R^2) > delta in floating point;
    constant reference v: sum R^2 = N v^2 (closed form); black reference: any change passes."""
    rng = np.random.default_rng(24)
    N = 30000
    for v in [0, 1, 100, 255]:
        assert orc.sum_sq(np.full(N, v, np.uint8)) == N * v * v
    assert orc.nrmse_threshold(0.5, 0) == 0
    for _ in range(200):
        ref = rng.integers(0, 256, N, dtype=np.uint8)
        Q = orc.sum_sq(ref)
        delta = float(rng.uniform(0.0, 1.5))
        T = orc.nrmse_threshold(delta, Q)
        for s in [int(rng.integers(0, 2 * Q)), T, T + 1]:
            val = math.sqrt(s / Q)
            if abs(val - delta) < 1e-9:
                continue
            assert orc.sdd_pass(s, T) == int(val > delta), (s, T, delta)


def test_sad_threshold_strict():
    for delta, T in [(0.0, 0), (264.0, 264), (264.5, 264), (265.0, 265)]:
        assert orc.sad_threshold(delta) == T
    assert orc.sdd_pass(265, orc.sad_threshold(264.99)) == 1
    assert orc.sdd_pass(265, orc.sad_threshold(265.0)) == 0


def test_previous_frame_reference_mode():
    """Reading Q25 ('previous' mode): frame t of a stream is compared with D100 of frame t-1 of the same
    stream, the first frame with the stream's reference. A static sequence is background after its first
    frame (P1 applied frame to frame); an A, B, A, B sequence has the same distance at every step (symmetry);
    two interleaved streams do not see each other's frames."""
    v = synth.Video(seed=77, width=200, height=120, period=6, on_len=3)
    W = 200
    a = synth.frame(v, 0, 0)
    b = synth.frame(v, 0, 3)  # a target frame (object planted)
    R = orc.reference(synth.frames(v, [0] * 4, list(range(4)), ref=True), W, 100, 100)
    p = synth.snm_weights(1, 0)
    n = 6

    def run(frames, sids, metric):
        return orc.filter_frames(frames, W, [R] * len(frames), [24.0 if metric != "sad" else 1000.0] * len(frames),
                                 [p] * len(frames), [0.2] * len(frames), [0.8] * len(frames), [0.5] * len(frames),
                                 run_snm=False, metrics=[metric] * len(frames),
                                 ref_modes=["previous"] * len(frames), stream_ids=sids)

    for metric in ["mse", "sad"]:
        r = run([a] * n, [0] * n, metric)
        assert (r["ssd"][1:] == 0).all() and (r["sdd_pass"][1:] == 0).all()
        assert r["ssd"][0] == orc.distance(metric, orc.box_downsample(a, W, 100, 100), R)
        r = run([a, b] * 3, [0] * n, metric)
        dab = orc.distance(metric, orc.box_downsample(a, W, 100, 100), orc.box_downsample(b, W, 100, 100))
        assert dab > 0 and (r["ssd"][1:] == dab).all() and (r["sdd_pass"][1:] == 1).all()
        assert np.array_equal(r["last_ref"][0], orc.box_downsample(b, W, 100, 100))
        # streams 0 and 1 interleaved, each static: only the first frame of each stream may differ from 0
        r = run([a, b, a, b, a, b], [0, 1, 0, 1, 0, 1], metric)
        assert (r["ssd"][2:] == 0).all()


# ------------------------------------------------------------------ f1: T-YOLO + NumberofObjects (P14-P17)

def test_p14_tyolo_count_hand_example():
    g = _gold("p14_tyolo_count.json")
    ln = {"0": 0.0, "ln3": math.log(3), "-ln3": -math.log(3), "ln19": math.log(19),
          "ln(19*0.4/0.6)": math.log(19 * 0.4 / 0.6)}
    out = np.zeros((1, 1, 125))
    for b in range(5):
        out[0, 0, 25 * b + 4] = ln[g["objectness"][b]]
        out[0, 0, 25 * b + 5 + 6] = ln[g["target_logit"][b]]
    s = orc.tyolo_scores(out, 6)[0]
    assert np.allclose(s, g["expected_scores"], rtol=0, atol=1e-12)
    # box 3 sits at 0.2 up to rounding of the logs: the hand count avoids relying on which side it lands
    assert orc.tyolo_count(out, 6, 0.2 + 1e-9) == g["expected_count_at_0.2"]
    assert orc.tyolo_count(out, 6, 0.1) == g["expected_count_at_0.1"]
    assert orc.tyolo_count(out, 7, 0.2) == 0  # another class: 1/38 at best


def test_p15_resize_upsampling_and_pool_s1_hand():
    g = _gold("p15_resize_pool.json")
    f, W = _frame_from_channel0(g["resize"]["channel0"])
    d = orc.resize(f, W, *g["resize"]["grid"])
    assert d[:, :, 0].tolist() == g["resize"]["expected_channel0"]
    x = np.asarray(g["pool_s1"]["input"], np.float64)[None]
    assert orc.maxpool2_s1(x)[0].tolist() == g["pool_s1"]["expected"]


@pytest.mark.parametrize("W,H,D", [(640, 360, 100), (1280, 720, 416), (1920, 1080, 416), (416, 416, 416)])
def test_resize_reduces_to_box_downsample_when_downscaling(W, H, D):
    f = np.random.default_rng(W).integers(0, 256, size=(H, 3 * W), dtype=np.uint8)
    if W >= D and H >= D:
        assert np.array_equal(orc.resize(f, W, D, D), orc.box_downsample(f, W, D, D))


def test_resize_mixed_up_and_down():
    """640x360 -> 416x416: x downsamples (boxes of 1-2 px), y upsamples (one source row per cell, row
    floor(j*360/416)); checked against a brute-force restatement on both axes."""
    W, H, D = 640, 360, 416
    f = np.random.default_rng(1).integers(0, 256, size=(H, 3 * W), dtype=np.uint8)
    got = orc.resize(f, W, D, D)
    img = f.reshape(H, W, 3).astype(np.int64)
    for j in [0, 1, 2, 207, 415]:
        y = j * H // D
        for i in [0, 1, 100, 415]:
            x0, x1 = i * W // D, (i + 1) * W // D
            s = img[y, x0:x1].sum(axis=0)
            n = x1 - x0
            assert (got[j, i] == (2 * s + n) // (2 * n)).all()


def test_leaky_closed_form():
    v = np.array([-2.0, -0.5, 0.0, 0.25, 3.0])
    assert orc.leaky(v).tolist() == [-0.2, -0.05, 0.0, 0.25, 3.0]


def _torch_tyolo(img, params, bf16=False):
    """T-YOLO restated with torch fp64 library ops (conv2d, leaky_relu, max_pool2d) — independent of the oracle."""
    import torch
    import torch.nn.functional as F
    from synth.synth import TYOLO_LAYERS
    x = torch.from_numpy(img.astype(np.float64) / 256.0).permute(2, 0, 1)[None]
    p = torch.from_numpy(params.astype(np.float64))
    o = 0
    pools = [1, 1, 1, 1, 1, 2, 0, 0, 0]
    for i, (cin, cout, k) in enumerate(TYOLO_LAYERS):
        w = p[o:o + cout * cin * k * k].reshape(cout, cin, k, k)
        o += w.numel()
        b = p[o:o + cout]
        o += cout
        if bf16:
            w = w.to(torch.bfloat16).to(torch.float64)
        x = F.conv2d(x, w, b, padding=k // 2)
        if i < 8:
            x = F.leaky_relu(x, 0.1)
        if pools[i] == 1:
            x = F.max_pool2d(x, 2, 2)
        elif pools[i] == 2:
            x = F.max_pool2d(F.pad(x, (0, 1, 0, 1), value=-float("inf")), 2, 1)
        if bf16 and i < 8:
            x = x.to(torch.bfloat16).to(torch.float64)
    return x[0].permute(1, 2, 0).numpy()


@pytest.mark.parametrize("S", [32, 64])
def test_p16_tyolo_forward_vs_torch_fp64(S):
    from synth import synth as sy
    rng = np.random.default_rng(S)
    img = rng.integers(0, 256, size=(S, S, 3), dtype=np.uint8)
    params = sy.tyolo_weights(S)
    got = orc.tyolo_forward(img, params)
    want = _torch_tyolo(img, params)
    assert got.shape == (S // 32, S // 32, 125)
    assert np.allclose(got, want, rtol=1e-9, atol=1e-9)
    got_b = orc.tyolo_forward(img, params, bf16_emul=True)
    want_b = _torch_tyolo(img, params, bf16=True)
    assert np.allclose(got_b, want_b, rtol=0, atol=5e-2)  # bf16 rounding flips from summation order only
    assert np.median(np.abs(got_b - want_b)) < 1e-3


def test_p17_tyolo_zero_weight_closed_form():
    """All conv weights 0, biases b_l: every layer outputs leaky(b_l) per channel (pooling keeps constants), so
    the output is b9 + W9 . leaky(b8) at every cell."""
    from synth import synth as sy
    params = np.zeros(orc.tyolo_n_params(), np.float32)
    rng = np.random.default_rng(17)
    o = 0
    b8 = w9 = b9 = None
    for i, (cin, cout, k) in enumerate(sy.TYOLO_LAYERS):
        nw = cout * cin * k * k
        if i == 8:
            w9 = rng.normal(0, 0.05, size=(cout, cin)).astype(np.float32)
            params[o:o + nw] = w9.ravel()
        o += nw
        b = rng.normal(0, 1, size=cout).astype(np.float32)
        params[o:o + cout] = b
        o += cout
        if i == 7:
            b8 = b
        if i == 8:
            b9 = b
    img = rng.integers(0, 256, size=(64, 64, 3), dtype=np.uint8)
    got = orc.tyolo_forward(img, params)
    lb8 = np.where(b8 < 0, 0.1 * b8.astype(np.float64), b8.astype(np.float64))
    want = b9.astype(np.float64) + w9.astype(np.float64) @ lb8
    assert np.allclose(got, np.broadcast_to(want, got.shape), rtol=1e-12, atol=1e-12)


def test_tyolo_n_params_tiny_yolo_voc():
    """tiny-yolo-voc: 15,858,717 parameters (conv weights + folded BN biases), hand sum over the nine layers."""
    assert orc.tyolo_n_params() == 448 + 4640 + 18496 + 73856 + 295168 + 1180160 + 4719616 + 9438208 + 128125
    assert orc.tyolo_n_params() == 15_858_717
