"""Seeded synthetic inputs (workload generator only — none of the method's arithmetic).

Shared by the oracle tests and the GPU path, as DESIGN.md "Input recipe" states:

* frames / reference frames: ``ffsva_synth.h`` through the host library
  ``libffsva_synth.so`` (CPU) or the device library ``libffsva_synth_cuda.so``
  (fills HBM pools; byte-identical to the host one);
* SNM weights: SURVEY.md §8(c) Q14 init — conv W ~ N(0, 2/fan_in) (He), FC ~
  N(0, 9/F) (gain 3), biases 0, every weight rounded to a bf16-representable
  value (RNE) and handed over as fp32, so the fp64 oracle and the bf16 kernel
  see the same numbers.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
HOST_LIB = os.path.join(_HERE, "libffsva_synth.so")
CUDA_LIB = os.path.join(_HERE, "libffsva_synth_cuda.so")


class SynthParams(ctypes.Structure):
    _fields_ = [("seed", ctypes.c_uint64), ("width", ctypes.c_int32), ("height", ctypes.c_int32),
                ("period", ctypes.c_int32), ("on_len", ctypes.c_int32)]


@dataclass(frozen=True)
class Video:
    """One synthetic video shape: W x H RGB8, target schedule (period P, L_on on-frames)."""
    seed: int
    width: int
    height: int
    period: int = 300
    on_len: int = 30

    @property
    def tor(self) -> float:
        """Target-object ratio, Eq. (1)."""
        return self.on_len / self.period

    def params(self) -> SynthParams:
        return SynthParams(self.seed, self.width, self.height, self.period, self.on_len)


_host = None
_cuda = None


def host_lib():
    global _host
    if _host is None:
        if not os.path.exists(HOST_LIB):
            raise RuntimeError(f"{HOST_LIB} missing: run __graft_entry__.build()")
        lib = ctypes.CDLL(HOST_LIB)
        P = ctypes.POINTER(SynthParams)
        lib.ffsva_synth_frame.argtypes = [P, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32, ctypes.c_void_p,
                                          ctypes.c_int64]
        lib.ffsva_synth_frames.argtypes = [P, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32,
                                           ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64]
        lib.ffsva_synth_target.argtypes = [P, ctypes.c_int32, ctypes.c_int64]
        lib.ffsva_synth_target.restype = ctypes.c_int32
        lib.ffsva_synth_planted.argtypes = [P, ctypes.c_int32, ctypes.c_int64, ctypes.c_int64]
        lib.ffsva_synth_planted.restype = ctypes.c_int64
        lib.ffsva_synth_object.argtypes = [P, ctypes.c_int32, ctypes.c_int64, ctypes.c_void_p]
        _host = lib
    return _host


def cuda_lib():
    global _cuda
    if _cuda is None:
        if not os.path.exists(CUDA_LIB):
            raise RuntimeError(f"{CUDA_LIB} missing: run __graft_entry__.build()")
        lib = ctypes.CDLL(CUDA_LIB)
        lib.ffsva_synth_frames_cuda.argtypes = [ctypes.POINTER(SynthParams), ctypes.c_void_p, ctypes.c_void_p,
                                                ctypes.c_int32, ctypes.c_int32, ctypes.c_void_p, ctypes.c_int64,
                                                ctypes.c_int64, ctypes.c_void_p]
        lib.ffsva_synth_frames_cuda.restype = ctypes.c_int
        _cuda = lib
    return _cuda


def frame(video: Video, stream: int, t: int, ref: bool = False, pitch: int | None = None) -> np.ndarray:
    """Frame t of `stream` as a (H, pitch) uint8 array (pitch defaults to 3W; padding bytes are 0)."""
    pitch = 3 * video.width if pitch is None else pitch
    out = np.zeros((video.height, pitch), dtype=np.uint8)
    p = video.params()
    host_lib().ffsva_synth_frame(ctypes.byref(p), stream, t, int(ref), out.ctypes.data, pitch)
    return out


def frames(video: Video, streams, ts, ref: bool = False, pitch: int | None = None) -> np.ndarray:
    """Stack of frames (n, H, pitch) uint8 for (streams[i], ts[i])."""
    pitch = 3 * video.width if pitch is None else pitch
    s = np.ascontiguousarray(np.asarray(streams, dtype=np.int32))
    t = np.ascontiguousarray(np.asarray(ts, dtype=np.int64))
    out = np.zeros((len(s), video.height, pitch), dtype=np.uint8)
    p = video.params()
    host_lib().ffsva_synth_frames(ctypes.byref(p), s.ctypes.data, t.ctypes.data, len(s), int(ref), out.ctypes.data,
                                  video.height * pitch, pitch)
    return out


def is_target(video: Video, stream: int, t: int) -> bool:
    p = video.params()
    return bool(host_lib().ffsva_synth_target(ctypes.byref(p), stream, t))


def planted(video: Video, stream: int, t0: int, t1: int) -> int:
    p = video.params()
    return int(host_lib().ffsva_synth_planted(ctypes.byref(p), stream, t0, t1))


def object_rect(video: Video, stream: int, t: int):
    out = np.zeros(4, dtype=np.int32)
    p = video.params()
    host_lib().ffsva_synth_object(ctypes.byref(p), stream, t, out.ctypes.data)
    return tuple(int(v) for v in out)


def frames_cuda(video: Video, streams_dev, ts_dev, out_dev, frame_stride: int, pitch: int, ref: bool = False,
                stream_handle: int = 0) -> None:
    """Device generator: fill out_dev (device pointer) with frames (streams_dev[i], ts_dev[i]).

    streams_dev: int32 device pointer, ts_dev: int64 device pointer (n = len)."""
    n = int(streams_dev.numel())
    p = video.params()
    rc = cuda_lib().ffsva_synth_frames_cuda(ctypes.byref(p), streams_dev.data_ptr(), ts_dev.data_ptr(), n, int(ref),
                                            out_dev.data_ptr(), frame_stride, pitch, stream_handle)
    if rc != 0:
        raise RuntimeError(f"ffsva_synth_frames_cuda failed: {rc}")


# ---------------------------------------------------------------- SNM weights (Q14)

def to_bf16_values(x: np.ndarray) -> np.ndarray:
    """Round float32 values to the nearest bf16-representable value (RNE); returns float32."""
    b = np.ascontiguousarray(x, dtype=np.float32).view(np.uint32).astype(np.uint64)
    rounded = (b + 0x7FFF + ((b >> 16) & 1)) >> 16
    return (rounded.astype(np.uint32) << 16).view(np.float32)


def snm_n_params(c1: int = 16, c2: int = 32, h: int = 50, w: int = 50) -> int:
    """SURVEY.md §8(c) C6 packing size: 27c1 + c1 + 9c1c2 + c2 + F + 1, F = c2*floor(floor(h/2)/2)*floor(floor(w/2)/2)."""
    f = c2 * ((h // 2) // 2) * ((w // 2) // 2)
    return 27 * c1 + c1 + 9 * c1 * c2 + c2 + f + 1


def snm_weights(seed: int, stream: int, c1: int = 16, c2: int = 32, h: int = 50, w: int = 50,
                fc_gain: float = 3.0, bias_std: float = 0.0) -> np.ndarray:
    """Packed SNM params w1[c1][3][3][3], b1[c1], w2[c2][c1][3][3], b2[c2], wfc[F], bfc[1] (float32, bf16-exact)."""
    rng = np.random.default_rng([seed, 0x534E4D, stream])
    f = c2 * ((h // 2) // 2) * ((w // 2) // 2)
    w1 = rng.normal(0.0, np.sqrt(2.0 / 27.0), size=(c1, 3, 3, 3))
    w2 = rng.normal(0.0, np.sqrt(2.0 / (9.0 * c1)), size=(c2, c1, 3, 3))
    wfc = rng.normal(0.0, fc_gain / np.sqrt(f), size=(f,))
    b1 = rng.normal(0.0, bias_std, size=(c1,)) if bias_std else np.zeros(c1)
    b2 = rng.normal(0.0, bias_std, size=(c2,)) if bias_std else np.zeros(c2)
    bfc = rng.normal(0.0, bias_std, size=(1,)) if bias_std else np.zeros(1)
    packed = np.concatenate([w1.ravel(), b1, w2.ravel(), b2, wfc, bfc]).astype(np.float32)
    return to_bf16_values(packed)


# tiny-yolo-voc layer table (Cin, Cout, kernel): the shape of the random-init weights the T-YOLO stage takes
TYOLO_LAYERS = [(3, 16, 3), (16, 32, 3), (32, 64, 3), (64, 128, 3), (128, 256, 3), (256, 512, 3), (512, 1024, 3),
                (1024, 1024, 3), (1024, 125, 1)]


def tyolo_weights(seed: int, target_class: int = 6, class_bias: float = 3.0, bias_std: float = 0.05,
                  out_gain: float = 1.0) -> np.ndarray:
    """Seeded random T-YOLO params (no trained VOC weights exist here): per layer w[Cout][Cin][k][k] (He normal,
    N(0, 2/fan_in); the last layer N(0, out_gain^2/fan_in)) then b[Cout] (N(0, bias_std^2); the last layer 0 except
    +class_bias on target_class's logit of every box, so scores straddle the 0.2 threshold). float32, bf16-exact."""
    rng = np.random.default_rng([seed, 0x59_4F_4C_4F])
    parts = []
    for i, (cin, cout, k) in enumerate(TYOLO_LAYERS):
        fan = cin * k * k
        last = i == len(TYOLO_LAYERS) - 1
        std = out_gain / np.sqrt(fan) if last else np.sqrt(2.0 / fan)
        w = rng.standard_normal(size=cout * fan, dtype=np.float32) * np.float32(std)
        if last:
            b = np.zeros(cout, np.float32)
            for box in range(5):
                b[25 * box + 5 + target_class] = class_bias
        else:
            b = (rng.standard_normal(size=cout, dtype=np.float32) * np.float32(bias_std)).astype(np.float32)
        parts += [w, b]
    return to_bf16_values(np.concatenate(parts).astype(np.float32))
