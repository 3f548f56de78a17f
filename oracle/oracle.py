"""Python face of the C oracle (oracle/ffsva_oracle.c) — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's CPU-baseline leg
(``cpu_baseline`` and ``--impl reference``) import this module. It is ctypes
marshalling around the plain single-threaded C definitions plus
``filter_frames``, which applies them frame by frame in the paper's order
(SDD: downsample -> distance -> threshold; survivors in order,
L143; SNM -> Eq. (2) decision, L159-L165, L193).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

u8p = ctypes.c_void_p


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run __graft_entry__.build()")
        L = ctypes.CDLL(LIB_PATH)
        L.orc_box_downsample.argtypes = [u8p, ctypes.c_int32, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32,
                                         ctypes.c_int32, u8p]
        L.orc_reference.argtypes = [u8p, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32,
                                    ctypes.c_int64, ctypes.c_int32, ctypes.c_int32, u8p]
        L.orc_ssd.argtypes = [u8p, u8p, ctypes.c_int64]
        L.orc_ssd.restype = ctypes.c_uint64
        L.orc_threshold.argtypes = [ctypes.c_double, ctypes.c_int64]
        L.orc_threshold.restype = ctypes.c_uint64
        L.orc_sad.argtypes = [u8p, u8p, ctypes.c_int64]
        L.orc_sad.restype = ctypes.c_uint64
        L.orc_sum_sq.argtypes = [u8p, ctypes.c_int64]
        L.orc_sum_sq.restype = ctypes.c_uint64
        L.orc_sdd_pass.argtypes = [ctypes.c_uint64, ctypes.c_uint64]
        L.orc_sdd_pass.restype = ctypes.c_int32
        L.orc_compact.argtypes = [u8p, ctypes.c_int32, u8p]
        L.orc_compact.restype = ctypes.c_int32
        L.orc_round_bf16.argtypes = [ctypes.c_double]
        L.orc_round_bf16.restype = ctypes.c_double
        L.orc_conv3x3.argtypes = [u8p, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, u8p, u8p, ctypes.c_int32, u8p]
        L.orc_maxpool2.argtypes = [u8p, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, u8p]
        L.orc_snm_forward.argtypes = [u8p, ctypes.c_int32, ctypes.c_int32, u8p, ctypes.c_int32, ctypes.c_int32,
                                      ctypes.c_int32]
        L.orc_snm_forward.restype = ctypes.c_double
        L.orc_snm_n_params.argtypes = [ctypes.c_int32] * 4
        L.orc_snm_n_params.restype = ctypes.c_int64
        L.orc_tpre.argtypes = [ctypes.c_double] * 3
        L.orc_tpre.restype = ctypes.c_double
        L.orc_logit.argtypes = [ctypes.c_double]
        L.orc_logit.restype = ctypes.c_double
        L.orc_decide.argtypes = [ctypes.c_double, ctypes.c_double, ctypes.c_double, ctypes.c_double, u8p, u8p]
        L.orc_resize.argtypes = [u8p, ctypes.c_int32, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32,
                                 u8p]
        L.orc_conv1x1.argtypes = [u8p, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, u8p, u8p, ctypes.c_int32, u8p]
        L.orc_leaky.argtypes = [u8p, ctypes.c_int64]
        L.orc_maxpool2_s1.argtypes = [u8p, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, u8p]
        L.orc_tyolo_forward.argtypes = [u8p, ctypes.c_int32, u8p, ctypes.c_int32, u8p]
        L.orc_tyolo_forward.restype = ctypes.c_int32
        L.orc_tyolo_n_params.argtypes = []
        L.orc_tyolo_n_params.restype = ctypes.c_int64
        L.orc_tyolo_count.argtypes = [u8p, ctypes.c_int32, ctypes.c_int32, ctypes.c_double]
        L.orc_tyolo_count.restype = ctypes.c_int32
        _lib = L
    return _lib


def _c(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


def box_downsample(frame: np.ndarray, width: int, dw: int, dh: int) -> np.ndarray:
    """C1. frame: (H, pitch) uint8 with 3*width <= pitch. Returns (dh, dw, 3) uint8."""
    f = _c(frame, np.uint8)
    H, pitch = f.shape
    out = np.zeros((dh, dw, 3), dtype=np.uint8)
    lib().orc_box_downsample(f.ctypes.data, width, H, pitch, dw, dh, out.ctypes.data)
    return out


def reference(frames: np.ndarray, width: int, dw: int, dh: int) -> np.ndarray:
    """C2. frames: (K, H, pitch) uint8 background frames. Returns (dh, dw, 3) uint8."""
    f = _c(frames, np.uint8)
    K, H, pitch = f.shape
    out = np.zeros((dh, dw, 3), dtype=np.uint8)
    lib().orc_reference(f.ctypes.data, K, H * pitch, width, H, pitch, dw, dh, out.ctypes.data)
    return out


def ssd(a: np.ndarray, b: np.ndarray) -> int:
    """C3 sum of squared differences (u64)."""
    a = _c(a, np.uint8).ravel()
    b = _c(b, np.uint8).ravel()
    assert a.size == b.size
    return int(lib().orc_ssd(a.ctypes.data, b.ctypes.data, a.size))


def threshold(delta_diff: float, n_values: int) -> int:
    """C3 T = floor(delta_diff * N)."""
    return int(lib().orc_threshold(delta_diff, n_values))


def sad(a: np.ndarray, b: np.ndarray) -> int:
    """f3 sum of absolute differences (reading Q23)."""
    a = _c(a, np.uint8).ravel()
    b = _c(b, np.uint8).ravel()
    assert a.size == b.size
    return int(lib().orc_sad(a.ctypes.data, b.ctypes.data, a.size))


def sum_sq(a: np.ndarray) -> int:
    """f3 NRMSE normaliser: sum of squares of the reference image (reading Q24)."""
    a = _c(a, np.uint8).ravel()
    return int(lib().orc_sum_sq(a.ctypes.data, a.size))


def sad_threshold(delta_diff: float) -> int:
    """f3 SAD: pass iff SAD > delta_diff <=> SAD > floor(delta_diff) (reading Q23)."""
    return threshold(delta_diff, 1)


def nrmse_threshold(delta_diff: float, ref_sum_sq: int) -> int:
    """f3 NRMSE = sqrt(SSD / sum R^2) (reading Q24). NRMSE > delta <=> SSD > delta^2 * sum R^2
    <=> SSD > floor(delta^2 * sum R^2), delta taken as the exact rational value of the double. Clamped to u64."""
    from fractions import Fraction
    if not delta_diff > 0:
        return 0
    t = (Fraction(delta_diff) ** 2 * ref_sum_sq).__floor__()
    return min(int(t), 2 ** 64 - 1)


def distance(metric: str, d100: np.ndarray, ref: np.ndarray) -> int:
    """The SDD distance numerator K1 reports in `ssd`: SSD for MSE and NRMSE, SAD for SAD."""
    return sad(d100, ref) if metric == "sad" else ssd(d100, ref)


def sdd_threshold(metric: str, delta_diff: float, ref: np.ndarray) -> int:
    """T of the strict test distance > T for each metric (readings Q5, Q23, Q24)."""
    if metric == "mse":
        return threshold(delta_diff, int(np.asarray(ref).size))
    if metric == "sad":
        return sad_threshold(delta_diff)
    if metric == "nrmse":
        return nrmse_threshold(delta_diff, sum_sq(ref))
    raise ValueError(metric)


def sdd_pass(ssd_value: int, T: int) -> int:
    return int(lib().orc_sdd_pass(ssd_value, T))


def compact(pass_mask) -> np.ndarray:
    """C4 survivors in batch order."""
    p = _c(pass_mask, np.uint8)
    idx = np.zeros(max(1, p.size), dtype=np.int32)
    m = lib().orc_compact(p.ctypes.data, p.size, idx.ctypes.data)
    return idx[:m].copy()


def round_bf16(x: float) -> float:
    return float(lib().orc_round_bf16(x))


def conv3x3(inp: np.ndarray, w: np.ndarray, b: np.ndarray | None = None) -> np.ndarray:
    """C6 single conv layer. inp (C, H, W), w (K, C, 3, 3), b (K,) -> (K, H, W) float64."""
    x = _c(inp, np.float64)
    wt = _c(w, np.float64)
    C, H, W = x.shape
    K = wt.shape[0]
    out = np.zeros((K, H, W), dtype=np.float64)
    bb = _c(b, np.float64) if b is not None else None
    lib().orc_conv3x3(x.ctypes.data, C, H, W, wt.ctypes.data, bb.ctypes.data if bb is not None else None, K,
                      out.ctypes.data)
    return out


def maxpool2(inp: np.ndarray) -> np.ndarray:
    x = _c(inp, np.float64)
    C, H, W = x.shape
    out = np.zeros((C, H // 2, W // 2), dtype=np.float64)
    lib().orc_maxpool2(x.ctypes.data, C, H, W, out.ctypes.data)
    return out


def snm_n_params(h: int = 50, w: int = 50, c1: int = 16, c2: int = 32) -> int:
    return int(lib().orc_snm_n_params(h, w, c1, c2))


def snm_forward(d50: np.ndarray, params: np.ndarray, c1: int = 16, c2: int = 32, bf16_emul: bool = False) -> float:
    """C5 + C6. d50: (h, w, 3) uint8; params packed float32 (C6 order). Returns the fp64 logit."""
    d = _c(d50, np.uint8)
    h, w, _ = d.shape
    p = _c(params, np.float32)
    assert p.size == snm_n_params(h, w, c1, c2)
    return float(lib().orc_snm_forward(d.ctypes.data, h, w, p.ctypes.data, c1, c2, int(bf16_emul)))


def tpre(c_low: float, c_high: float, filter_degree: float) -> float:
    """PAPER.md L193 Eq. (2)."""
    return float(lib().orc_tpre(c_low, c_high, filter_degree))


def logit(t: float) -> float:
    return float(lib().orc_logit(t))


def decide(logit_value: float, c_low: float, c_high: float, filter_degree: float):
    """C7 -> (pass, class)."""
    p = np.zeros(1, dtype=np.uint8)
    c = np.zeros(1, dtype=np.uint8)
    lib().orc_decide(logit_value, c_low, c_high, filter_degree, p.ctypes.data, c.ctypes.data)
    return int(p[0]), int(c[0])


def filter_frames(frames, width: int, refs, deltas, snm_params, c_low, c_high, filter_degree,
                  sdd_grid=(100, 100), snm_grid=(50, 50), bf16_emul: bool = False, run_snm: bool = True,
                  metrics=None, ref_modes=None, stream_ids=None):
    """The whole cascade on a list of frames, one frame at a time (no batching: C8 says batching never
    changes per-frame results).

    frames[i]: (H, pitch) uint8; refs[i]: (sdd_h, sdd_w, 3) reference of frame i's stream; deltas[i]:
    delta_diff; snm_params[i]: packed params (or None); c_low/c_high/filter_degree: per-frame sequences.
    f3 variants (optional per-frame sequences): metrics[i] in {"mse", "sad", "nrmse"};
    ref_modes[i] in {"background", "previous"} with stream_ids[i]: in "previous" mode a frame is compared with
    the D100 of its stream's previous frame in list order, the first one with refs[i] (reading Q25).
    Returns dict of per-frame arrays: d100, d50, ssd, sdd_pass, survivor_idx, logit, snm_pass, snm_class, and
    last_ref: {stream id: reference after the list} for "previous"-mode streams."""
    n = len(frames)
    dw, dh = sdd_grid
    sw, sh = snm_grid
    metrics = metrics if metrics is not None else ["mse"] * n
    ref_modes = ref_modes if ref_modes is not None else ["background"] * n
    d100 = np.zeros((n, dh, dw, 3), np.uint8)
    d50 = np.zeros((n, sh, sw, 3), np.uint8)
    ssd_v = np.zeros(n, np.uint64)
    sp = np.zeros(n, np.uint8)
    last_ref = {}
    for i in range(n):
        d100[i] = box_downsample(frames[i], width, dw, dh)
        d50[i] = box_downsample(frames[i], width, sw, sh)
        ref = refs[i]
        if ref_modes[i] == "previous":
            ref = last_ref.get(stream_ids[i], refs[i])
            last_ref[stream_ids[i]] = d100[i]
        ssd_v[i] = distance(metrics[i], d100[i], ref)
        sp[i] = sdd_pass(int(ssd_v[i]), sdd_threshold(metrics[i], deltas[i], ref))
    surv = compact(sp)
    sidx = np.full(n, -1, np.int32)
    sidx[surv] = np.arange(surv.size, dtype=np.int32)
    lg = np.full(n, np.nan, np.float64)
    npass = np.zeros(n, np.uint8)
    ncls = np.zeros(n, np.uint8)
    if run_snm:
        for i in surv:
            lg[i] = snm_forward(d50[i], snm_params[i], bf16_emul=bf16_emul)
            npass[i], ncls[i] = decide(lg[i], c_low[i], c_high[i], filter_degree[i])
    return dict(d100=d100, d50=d50, ssd=ssd_v, sdd_pass=sp, survivors=surv, survivor_idx=sidx, logit=lg,
                snm_pass=npass, snm_class=ncls, last_ref=last_ref)


# ------------------------------------------------------------------ f1: T-YOLO + NumberofObjects (L169-L175, L195)

def resize(frame: np.ndarray, width: int, dw: int, dh: int) -> np.ndarray:
    """Q28 resize (C1 box when the frame is larger, one source pixel per cell when smaller). -> (dh, dw, 3) u8."""
    f = _c(frame, np.uint8)
    H, pitch = f.shape
    out = np.zeros((dh, dw, 3), dtype=np.uint8)
    lib().orc_resize(f.ctypes.data, width, H, pitch, dw, dh, out.ctypes.data)
    return out


def conv1x1(inp: np.ndarray, w: np.ndarray, b: np.ndarray | None = None) -> np.ndarray:
    x = _c(inp, np.float64)
    wt = _c(w, np.float64)
    C, H, W = x.shape
    K = wt.shape[0]
    out = np.zeros((K, H, W), dtype=np.float64)
    bb = _c(b, np.float64) if b is not None else None
    lib().orc_conv1x1(x.ctypes.data, C, H, W, wt.ctypes.data, bb.ctypes.data if bb is not None else None, K,
                      out.ctypes.data)
    return out


def leaky(v: np.ndarray) -> np.ndarray:
    x = np.array(v, dtype=np.float64, copy=True, order="C")
    lib().orc_leaky(x.ctypes.data, x.size)
    return x


def maxpool2_s1(inp: np.ndarray) -> np.ndarray:
    x = _c(inp, np.float64)
    C, H, W = x.shape
    out = np.zeros_like(x)
    lib().orc_maxpool2_s1(x.ctypes.data, C, H, W, out.ctypes.data)
    return out


def tyolo_n_params() -> int:
    return int(lib().orc_tyolo_n_params())


def tyolo_forward(img: np.ndarray, params: np.ndarray, bf16_emul: bool = False) -> np.ndarray:
    """T-YOLO on an (S, S, 3) u8 image (S = 416, or any multiple of 32). Returns (S/32, S/32, 125) float64."""
    im = _c(img, np.uint8)
    S = im.shape[0]
    assert im.shape == (S, S, 3)
    p = _c(params, np.float32)
    assert p.size == tyolo_n_params()
    out = np.zeros((S // 32, S // 32, 125), np.float64)
    assert lib().orc_tyolo_forward(im.ctypes.data, S, p.ctypes.data, int(bf16_emul), out.ctypes.data) == 0
    return out


def tyolo_count(out: np.ndarray, target_class: int, thresh: float = 0.2) -> int:
    """L171 + Q31: boxes whose sigmoid(objectness) * softmax(classes)[target] exceeds thresh."""
    o = _c(out, np.float64)
    return int(lib().orc_tyolo_count(o.ctypes.data, o.size // 125, target_class, thresh))


def tyolo_scores(out: np.ndarray, target_class: int) -> np.ndarray:
    """Per-box scores (cells x 5) by the same definition, for near-threshold exemptions in parity tests."""
    o = np.asarray(out, np.float64).reshape(-1, 5, 25)
    cls = o[:, :, 5:]
    e = np.exp(cls - cls.max(axis=2, keepdims=True))
    return 1.0 / (1.0 + np.exp(-o[:, :, 4])) * e[:, :, target_class] / e.sum(axis=2)
