"""Thin Python binding of the C-ABI in include/ffsva.h (ctypes argument marshalling only).

Every function named ``ffsva_*`` here is the C entry point of the same name; every step of the filter
cascade runs in the library's sm_100a kernels (paper_conf_icpp_zhangcjzly18_b200/lib/libffsva.so). There is
no CPU fallback: if the library is missing this module raises at import of the library, and on a machine
without a B200 every compute call fails with FFSVA_ECUDA.

The small convenience layer (``Context``, ``Stream``, ``PreparedBatch``) converts torch tensors / numpy
arrays to pointers and results to numpy arrays.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("FFSVA_LIB", os.path.join(_HERE, "lib", "libffsva.so"))  # FFSVA_LIB: A/B builds

FFSVA_OK, FFSVA_EINVAL, FFSVA_ENOMEM, FFSVA_ECUDA, FFSVA_ESTATE, FFSVA_EAGAIN, FFSVA_EDEVICE = 0, -1, -2, -3, -4, -5, -6
STATUS_NAMES = {0: "FFSVA_OK", -1: "FFSVA_EINVAL", -2: "FFSVA_ENOMEM", -3: "FFSVA_ECUDA", -4: "FFSVA_ESTATE",
                -5: "FFSVA_EAGAIN", -6: "FFSVA_EDEVICE"}
STAT_NAMES = (["frames", "sdd_pass", "snm_pass", "ssd_sum", "class0", "class1", "class2", "snm_batches", "decided",
               "lat_sum_us"] + [f"lat_bin{k}" for k in range(14)])  # include/ffsva.h FFSVA_STAT_*
LAT_BIN0 = 10
# latency bin k covers [LAT_EDGES_MS[k], LAT_EDGES_MS[k + 1]) milliseconds (bin 0 < 1 ms, bin 13 >= 4096 ms)
LAT_EDGES_MS = [0.0] + [float(2 ** (k - 1)) for k in range(1, 14)] + [float("inf")]
NSTAT = len(STAT_NAMES)

# Every symbol include/ffsva.h declares (checked by tests/test_abi.py).
EXPORTS = ["ffsva_open_stream", "ffsva_set_reference", "ffsva_snm_load", "ffsva_filter_batch",
           "ffsva_filter_batch_host", "ffsva_batch_prepare", "ffsva_batch_launch", "ffsva_batch_fetch",
           "ffsva_batch_device_outputs", "ffsva_batch_destroy", "ffsva_batch_profile", "ffsva_sdd_batch",
           "ffsva_get_reference",
           "ffsva_stream_info", "ffsva_stats_copy", "ffsva_close", "ffsva_last_error", "ffsva_kernel_launches",
           "ffsva_version", "ffsva_sched_create", "ffsva_sched_push", "ffsva_sched_tick", "ffsva_sched_depth",
           "ffsva_sched_destroy", "ffsva_sched_set_policy", "ffsva_sched_set_pipeline", "ffsva_stream_image_bytes",
           "ffsva_stream_export",
           "ffsva_stream_import", "ffsva_sched_stream_load", "ffsva_sched_detach", "ffsva_tyolo_load",
           "ffsva_tyolo_run", "ffsva_tyolo_layer_output", "ffsva_tyolo_profile", "ffsva_tyolo_destroy",
           "ffsva_sched_set_tyolo", "ffsva_sched_inspect"]


class StreamDesc(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("width", ctypes.c_int32), ("height", ctypes.c_int32),
                ("row_pitch", ctypes.c_int64), ("sdd_w", ctypes.c_int32), ("sdd_h", ctypes.c_int32),
                ("snm_w", ctypes.c_int32), ("snm_h", ctypes.c_int32), ("delta_diff", ctypes.c_double),
                ("c_low", ctypes.c_float), ("c_high", ctypes.c_float), ("filter_degree", ctypes.c_float),
                ("snm_batch", ctypes.c_int32), ("q_sdd", ctypes.c_int32), ("q_snm", ctypes.c_int32),
                ("distance", ctypes.c_int32), ("ref_mode", ctypes.c_int32),
                ("number_of_objects", ctypes.c_int32), ("target_class", ctypes.c_int32), ("q_tyolo", ctypes.c_int32)]


# ffsva_distance / ffsva_ref_mode (include/ffsva.h)
DISTANCES = {"mse": 0, "sad": 1, "nrmse": 2}
REF_MODES = {"background": 0, "previous": 1}


class SnmDesc(ctypes.Structure):
    _fields_ = [("c1", ctypes.c_int32), ("c2", ctypes.c_int32)]


class Frame(ctypes.Structure):
    _fields_ = [("stream", ctypes.c_void_p), ("pixels", ctypes.c_void_p), ("frame_no", ctypes.c_int64)]


class Result(ctypes.Structure):
    _fields_ = [("ssd", ctypes.c_uint64), ("sdd_pass", ctypes.c_uint8), ("snm_pass", ctypes.c_uint8),
                ("snm_class", ctypes.c_uint8), ("tyolo_pass", ctypes.c_uint8), ("logit", ctypes.c_float),
                ("survivor_idx", ctypes.c_int32), ("tyolo_count", ctypes.c_int32), ("reserved", ctypes.c_int32)]


RESULT_DTYPE = np.dtype([("ssd", "<u8"), ("sdd_pass", "u1"), ("snm_pass", "u1"), ("snm_class", "u1"),
                         ("tyolo_pass", "u1"), ("logit", "<f4"), ("survivor_idx", "<i4"), ("tyolo_count", "<i4"),
                         ("reserved", "<i4")], align=True)
assert RESULT_DTYPE.itemsize == ctypes.sizeof(Result) == 32

EVENT_DTYPE = np.dtype([("stream", "<u8"), ("frame_no", "<i8"), ("result", RESULT_DTYPE)], align=True)


class TickInfo(ctypes.Structure):
    _fields_ = [("admitted", ctypes.c_int32), ("sdd_pass", ctypes.c_int32), ("snm_scored", ctypes.c_int32),
                ("snm_batches", ctypes.c_int32), ("sdd_blocked", ctypes.c_int32), ("sdd_queued", ctypes.c_int64),
                ("snm_queued", ctypes.c_int64), ("events_pending", ctypes.c_int64), ("sdd_ms", ctypes.c_float),
                ("snm_ms", ctypes.c_float), ("host_ms", ctypes.c_float), ("pad", ctypes.c_int32),
                ("tyolo_scored", ctypes.c_int32), ("snm_blocked", ctypes.c_int32), ("tyolo_queued", ctypes.c_int64),
                ("tyolo_ms", ctypes.c_float), ("pad2", ctypes.c_int32)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class StreamLoad(ctypes.Structure):
    """ffsva_stream_load: per-stream overload signals of the online runtime."""
    _fields_ = [("sdd_depth", ctypes.c_int32), ("snm_depth", ctypes.c_int32), ("max_sdd", ctypes.c_int32),
                ("max_snm", ctypes.c_int32), ("pushed", ctypes.c_uint64), ("refused", ctypes.c_uint64),
                ("sdd_blocked", ctypes.c_uint64), ("tyolo_depth", ctypes.c_int32), ("max_tyolo", ctypes.c_int32),
                ("snm_blocked", ctypes.c_uint64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


IMAGE_DESC_OFFSET = 8  # ffsva_stream_desc inside a stream image header (after magic, version)

_lib = None


def lib():
    """Load libffsva.so (fails loudly if the extension was not built: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: run `python __graft_entry__.py` (build) first; "
                               "the filter cascade has no CPU fallback")
        L = ctypes.CDLL(LIB_PATH)
        vp, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
        sig = {
            "ffsva_open_stream": [ctypes.POINTER(StreamDesc), ctypes.POINTER(vp)],
            "ffsva_set_reference": [vp, vp, i32, i64],
            "ffsva_snm_load": [vp, ctypes.POINTER(SnmDesc), vp, i64],
            "ffsva_filter_batch": [vp, i32, vp, vp],
            "ffsva_filter_batch_host": [vp, i32, vp, vp],
            "ffsva_batch_prepare": [vp, i32, ctypes.POINTER(vp)],
            "ffsva_batch_launch": [vp, vp],
            "ffsva_batch_fetch": [vp, vp, vp],
            "ffsva_batch_device_outputs": [vp] + [ctypes.POINTER(vp)] * 7 + [ctypes.POINTER(i64), ctypes.POINTER(vp)],
            "ffsva_batch_destroy": [vp],
            "ffsva_batch_profile": [vp, i32, i32, vp, vp],
            "ffsva_sdd_batch": [vp, i32, vp, vp, vp, vp, vp],
            "ffsva_get_reference": [vp, vp],
            "ffsva_stream_info": [vp, ctypes.POINTER(i32), ctypes.POINTER(i32)],
            "ffsva_stats_copy": [i32, vp, i32, ctypes.POINTER(i32), i32, i32, vp],
            "ffsva_close": [vp],
            "ffsva_sched_create": [i32, i32, i32, ctypes.POINTER(vp)],
            "ffsva_sched_push": [vp, vp, i32, vp],
            "ffsva_sched_tick": [vp, vp, vp, i32, ctypes.POINTER(i32), ctypes.POINTER(TickInfo)],
            "ffsva_sched_depth": [vp, vp, ctypes.POINTER(i32), ctypes.POINTER(i32)],
            "ffsva_sched_destroy": [vp],
            "ffsva_sched_set_policy": [vp, i32],
            "ffsva_sched_set_pipeline": [vp, i32],
            "ffsva_stream_image_bytes": [vp, ctypes.POINTER(i64)],
            "ffsva_stream_export": [vp, vp, i64, i32, vp],
            "ffsva_stream_import": [i32, vp, i64, i32, ctypes.POINTER(vp)],
            "ffsva_sched_stream_load": [vp, vp, i32, ctypes.POINTER(StreamLoad)],
            "ffsva_sched_detach": [vp, vp],
            "ffsva_tyolo_load": [i32, vp, i64, ctypes.POINTER(vp)],
            "ffsva_tyolo_run": [vp, vp, i32, i32, ctypes.c_float, i32, vp, vp, vp, vp],
            "ffsva_tyolo_layer_output": [vp, vp, i32, i32, vp, vp],
            "ffsva_tyolo_profile": [vp, vp, i32, i32, vp, vp],
            "ffsva_tyolo_destroy": [vp],
            "ffsva_sched_set_tyolo": [vp, vp, i32, ctypes.c_float],
            "ffsva_sched_inspect": [vp, vp, vp, vp, i32, ctypes.POINTER(i32)],
        }
        for name, args in sig.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = ctypes.c_int
        L.ffsva_last_error.restype = ctypes.c_char_p
        L.ffsva_last_error.argtypes = []
        L.ffsva_version.restype = ctypes.c_char_p
        L.ffsva_version.argtypes = []
        L.ffsva_kernel_launches.restype = ctypes.c_uint64
        L.ffsva_kernel_launches.argtypes = []
        _lib = L
    return _lib


class FfsvaError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = lib().ffsva_last_error().decode()
        super().__init__(f"{where}: {STATUS_NAMES.get(status, status)}: {msg}")


def _check(status: int, where: str) -> None:
    if status != FFSVA_OK:
        raise FfsvaError(status, where)


# ------------------------------------------------------------------ C entry points, same names

def ffsva_open_stream(desc: StreamDesc):
    h = ctypes.c_void_p()
    _check(lib().ffsva_open_stream(ctypes.byref(desc), ctypes.byref(h)), "ffsva_open_stream")
    return h.value


def ffsva_set_reference(stream, frames_ptr: int, k: int, frame_stride: int) -> None:
    _check(lib().ffsva_set_reference(stream, frames_ptr, k, frame_stride), "ffsva_set_reference")


def ffsva_snm_load(stream, params: np.ndarray, c1: int = 16, c2: int = 32) -> None:
    p = np.ascontiguousarray(params, dtype=np.float32)
    d = SnmDesc(c1, c2)
    _check(lib().ffsva_snm_load(stream, ctypes.byref(d), p.ctypes.data, p.size), "ffsva_snm_load")


def _frames_array(frames):
    arr = (Frame * max(1, len(frames)))()
    for i, (s, ptr, no) in enumerate(frames):
        arr[i].stream = s
        arr[i].pixels = ptr
        arr[i].frame_no = no
    return arr


def ffsva_filter_batch(frames, cuda_stream: int = 0, host: bool = False) -> np.ndarray:
    """frames: list of (stream handle, pixels pointer, frame_no). Returns a RESULT_DTYPE array."""
    n = len(frames)
    arr = _frames_array(frames)
    out = np.zeros(max(1, n), dtype=RESULT_DTYPE)
    fn = lib().ffsva_filter_batch_host if host else lib().ffsva_filter_batch
    _check(fn(arr, n, out.ctypes.data, cuda_stream), "ffsva_filter_batch_host" if host else "ffsva_filter_batch")
    return out[:n]


def ffsva_sdd_batch(frames, sdd_w: int, sdd_h: int, want_d100: bool = True, cuda_stream: int = 0):
    n = len(frames)
    arr = _frames_array(frames)
    d100 = np.zeros((max(1, n), sdd_h, sdd_w, 3), np.uint8) if want_d100 else None
    d50 = np.zeros((max(1, n), sdd_h // 2, sdd_w // 2, 3), np.uint8)
    ssd = np.zeros(max(1, n), np.uint64)
    ps = np.zeros(max(1, n), np.uint8)
    _check(lib().ffsva_sdd_batch(arr, n, d100.ctypes.data if want_d100 else None, d50.ctypes.data,
                                 ssd.ctypes.data, ps.ctypes.data, cuda_stream), "ffsva_sdd_batch")
    return dict(d100=d100[:n] if want_d100 else None, d50=d50[:n], ssd=ssd[:n], sdd_pass=ps[:n])


def ffsva_batch_prepare(frames):
    arr = _frames_array(frames)
    h = ctypes.c_void_p()
    _check(lib().ffsva_batch_prepare(arr, len(frames), ctypes.byref(h)), "ffsva_batch_prepare")
    return h.value


def ffsva_batch_launch(batch, cuda_stream: int) -> None:
    _check(lib().ffsva_batch_launch(batch, cuda_stream), "ffsva_batch_launch")


def ffsva_batch_fetch(batch, n: int | None, cuda_stream: int):
    if n is None:
        _check(lib().ffsva_batch_fetch(batch, None, cuda_stream), "ffsva_batch_fetch")
        return None
    out = np.zeros(max(1, n), dtype=RESULT_DTYPE)
    _check(lib().ffsva_batch_fetch(batch, out.ctypes.data, cuda_stream), "ffsva_batch_fetch")
    return out[:n]


def ffsva_batch_device_outputs(batch) -> dict:
    ptrs = [ctypes.c_void_p() for _ in range(7)]
    stride = ctypes.c_int64()
    cnt = ctypes.c_void_p()
    _check(lib().ffsva_batch_device_outputs(batch, *[ctypes.byref(p) for p in ptrs], ctypes.byref(stride),
                                            ctypes.byref(cnt)), "ffsva_batch_device_outputs")
    names = ["ssd", "sdd_pass", "survivor_idx", "logit", "snm_pass", "snm_class", "d50"]
    d = {k: p.value for k, p in zip(names, ptrs)}
    d["d50_stride"] = stride.value
    d["n_survivors"] = cnt.value
    return d


def ffsva_batch_destroy(batch) -> None:
    _check(lib().ffsva_batch_destroy(batch), "ffsva_batch_destroy")


def ffsva_batch_profile(batches, iters: int, cuda_stream: int) -> list:
    """Mean device ms per launch of [K1, K3, K4] over iters passes of the prepared batches."""
    arr = (ctypes.c_void_p * len(batches))(*batches)
    ms = (ctypes.c_float * 3)()
    _check(lib().ffsva_batch_profile(arr, len(batches), iters, ms, cuda_stream), "ffsva_batch_profile")
    return [float(x) for x in ms]


def ffsva_get_reference(stream, sdd_w: int, sdd_h: int) -> np.ndarray:
    out = np.zeros((sdd_h, sdd_w, 3), np.uint8)
    _check(lib().ffsva_get_reference(stream, out.ctypes.data), "ffsva_get_reference")
    return out


def ffsva_stream_info(stream):
    slot, dev = ctypes.c_int32(), ctypes.c_int32()
    _check(lib().ffsva_stream_info(stream, ctypes.byref(slot), ctypes.byref(dev)), "ffsva_stream_info")
    return slot.value, dev.value


def ffsva_stats_copy(device: int, dst_ptr: int, max_slots: int, dst_is_host: bool, reset: bool = False,
                     cuda_stream: int = 0) -> int:
    slots = ctypes.c_int32()
    _check(lib().ffsva_stats_copy(device, dst_ptr, max_slots, ctypes.byref(slots), int(dst_is_host), int(reset),
                                  cuda_stream), "ffsva_stats_copy")
    return slots.value


def ffsva_close(stream) -> None:
    _check(lib().ffsva_close(stream), "ffsva_close")


def ffsva_kernel_launches() -> int:
    return int(lib().ffsva_kernel_launches())


def ffsva_version() -> str:
    return lib().ffsva_version().decode()


# ------------------------------------------------------------------ convenience layer

def _stream_handle(stream):
    """torch.cuda.Stream / int / None -> cudaStream_t value."""
    if stream is None:
        return 0
    if isinstance(stream, int):
        return stream
    return int(stream.cuda_stream)


class Stream:
    """One camera stream (per-stream SDD + SNM)."""

    def __init__(self, ctx: "Context", desc: StreamDesc):
        self.ctx = ctx
        self.desc = desc
        self.handle = ffsva_open_stream(desc)
        self.slot, self.device = ffsva_stream_info(self.handle)

    def set_reference(self, frames, k: int | None = None, frame_stride: int | None = None) -> None:
        """frames: torch tensor (device or host) or numpy array of k background frames (k, H, pitch)."""
        if isinstance(frames, np.ndarray):
            frames = np.ascontiguousarray(frames)
            k = frames.shape[0] if k is None else k
            stride = frames[0].nbytes if frame_stride is None else frame_stride
            ffsva_set_reference(self.handle, frames.ctypes.data, k, stride)
        else:
            frames = frames.contiguous()
            k = frames.shape[0] if k is None else k
            stride = frames[0].numel() * frames.element_size() if frame_stride is None else frame_stride
            ffsva_set_reference(self.handle, frames.data_ptr(), k, stride)

    def snm_load(self, params: np.ndarray) -> None:
        ffsva_snm_load(self.handle, params)

    def reference(self) -> np.ndarray:
        return ffsva_get_reference(self.handle, self.desc.sdd_w, self.desc.sdd_h)

    def image_bytes(self) -> int:
        n = ctypes.c_int64()
        _check(lib().ffsva_stream_image_bytes(self.handle, ctypes.byref(n)), "ffsva_stream_image_bytes")
        return n.value

    def export(self, out=None, stream=None):
        """The stream's image (f2 re-forwarding): a numpy uint8 array (host), or written into
        `out`, a uint8 torch tensor (device tensors must live on the stream's device). Returns the buffer."""
        n = self.image_bytes()
        if out is None:
            out = np.zeros(n, np.uint8)
        if isinstance(out, np.ndarray):
            assert out.dtype == np.uint8 and out.flags["C_CONTIGUOUS"]
            ptr, cap, host = out.ctypes.data, out.nbytes, 1
        else:
            ptr, cap, host = out.data_ptr(), out.numel() * out.element_size(), 0 if out.is_cuda else 1
        _check(lib().ffsva_stream_export(self.handle, ptr, cap, host, _stream_handle(stream)), "ffsva_stream_export")
        return out

    def close(self) -> None:
        if self.handle:
            ffsva_close(self.handle)
            self.handle = None


class Context:
    """Per-device convenience wrapper; the device context itself lives inside the library."""

    def __init__(self, device=0):
        self.device = device.index if hasattr(device, "index") and device.index is not None else int(
            getattr(device, "index", device) or 0)
        self.streams: list[Stream] = []

    def open_stream(self, width: int, height: int, row_pitch: int | None = None, delta_diff: float = 24.0,
                    c_low: float = 0.2, c_high: float = 0.8, filter_degree: float = 0.5, snm_batch: int = 30,
                    q_sdd: int = 2, q_snm: int = 10, sdd=(100, 100), distance: str = "mse",
                    ref_mode: str = "background", number_of_objects: int = 1, target_class: int = 6,
                    q_tyolo: int = 2) -> Stream:
        d = StreamDesc(self.device, width, height, 3 * width if row_pitch is None else row_pitch, sdd[0], sdd[1],
                       sdd[0] // 2, sdd[1] // 2, delta_diff, c_low, c_high, filter_degree, snm_batch, q_sdd, q_snm,
                       DISTANCES[distance], REF_MODES[ref_mode], number_of_objects, target_class, q_tyolo)
        s = Stream(self, d)
        self.streams.append(s)
        return s

    @staticmethod
    def _frames(items):
        out = []
        for s, px, no in items:
            ptr = px if isinstance(px, int) else (px.ctypes.data if isinstance(px, np.ndarray) else px.data_ptr())
            out.append((s.handle, ptr, no))
        return out

    def filter_batch(self, items, stream=None, host: bool = False) -> dict:
        """items: list of (Stream, pixels tensor/pointer, frame_no). Returns dict of per-frame numpy arrays."""
        r = ffsva_filter_batch(self._frames(items), _stream_handle(stream), host=host)
        return {k: r[k].copy() for k in ("ssd", "sdd_pass", "snm_pass", "snm_class", "logit", "survivor_idx")}

    def sdd_batch(self, items, want_d100: bool = True, stream=None) -> dict:
        s0 = items[0][0].desc
        return ffsva_sdd_batch(self._frames(items), s0.sdd_w, s0.sdd_h, want_d100, _stream_handle(stream))

    def prepare(self, items) -> "PreparedBatch":
        return PreparedBatch(self._frames(items))

    def stats(self, max_slots: int = 1024, reset: bool = False) -> np.ndarray:
        out = np.zeros((max_slots, NSTAT), np.uint64)
        slots = ffsva_stats_copy(self.device, out.ctypes.data, max_slots, True, reset)
        return out[:min(slots, max_slots)]

    def close(self) -> None:
        for s in self.streams:
            s.close()
        self.streams = []

    def import_stream(self, image) -> Stream:
        """Open a stream on this device from an image made by Stream.export (numpy host array or uint8 torch
        tensor on this device)."""
        if isinstance(image, np.ndarray):
            buf = np.ascontiguousarray(image, dtype=np.uint8)
            ptr, n, host, hdr = buf.ctypes.data, buf.nbytes, 1, buf[:256].tobytes()
        else:
            ptr, n = image.data_ptr(), image.numel()
            host = 0 if image.is_cuda else 1
            hdr = image[:256].cpu().numpy().tobytes()
        h = ctypes.c_void_p()
        _check(lib().ffsva_stream_import(self.device, ptr, n, host, ctypes.byref(h)), "ffsva_stream_import")
        desc = StreamDesc.from_buffer_copy(hdr, IMAGE_DESC_OFFSET)
        desc.device = self.device
        st = Stream.__new__(Stream)
        st.ctx, st.desc, st.handle = self, desc, h.value
        st.slot, st.device = ffsva_stream_info(st.handle)
        self.streams.append(st)
        return st


def ffsva_sched_create(device: int, max_frames_per_tick: int, snm_slots: int):
    h = ctypes.c_void_p()
    _check(lib().ffsva_sched_create(device, max_frames_per_tick, snm_slots, ctypes.byref(h)), "ffsva_sched_create")
    return h.value


def ffsva_sched_push(sched, frames) -> np.ndarray:
    """frames: list of (stream handle, device pointer, frame_no) or a structured array. Returns accepted (u8)."""
    arr = _frames_array(frames)
    acc = np.zeros(max(1, len(frames)), np.uint8)
    _check(lib().ffsva_sched_push(sched, arr, len(frames), acc.ctypes.data), "ffsva_sched_push")
    return acc[:len(frames)]


def ffsva_sched_push_array(sched, frames: np.ndarray) -> np.ndarray:
    """Vectorised push: frames is a FRAME_DTYPE array (stream handle, pixels pointer, frame_no)."""
    f = np.ascontiguousarray(frames, dtype=FRAME_DTYPE)
    acc = np.zeros(max(1, f.size), np.uint8)
    _check(lib().ffsva_sched_push(sched, f.ctypes.data, f.size, acc.ctypes.data), "ffsva_sched_push")
    return acc[:f.size]


def ffsva_sched_tick(sched, cuda_stream: int, cap: int):
    ev = np.zeros(max(1, cap), EVENT_DTYPE)
    n = ctypes.c_int32()
    info = TickInfo()
    _check(lib().ffsva_sched_tick(sched, cuda_stream, ev.ctypes.data, cap, ctypes.byref(n), ctypes.byref(info)),
           "ffsva_sched_tick")
    return ev[:n.value], info.as_dict()


def ffsva_sched_depth(sched, stream):
    a, b = ctypes.c_int32(), ctypes.c_int32()
    _check(lib().ffsva_sched_depth(sched, stream, ctypes.byref(a), ctypes.byref(b)), "ffsva_sched_depth")
    return a.value, b.value


def ffsva_sched_destroy(sched) -> None:
    _check(lib().ffsva_sched_destroy(sched), "ffsva_sched_destroy")


# ffsva_batch_policy (include/ffsva.h; §4.3.2, §5.4)
BATCH_POLICIES = {"dynamic": 0, "feedback": 1, "static": 2}


def ffsva_sched_set_policy(sched, policy: str) -> None:
    _check(lib().ffsva_sched_set_policy(sched, BATCH_POLICIES[policy]), "ffsva_sched_set_policy")


FRAME_DTYPE = np.dtype([("stream", "<u8"), ("pixels", "<u8"), ("frame_no", "<i8")], align=True)


class Scheduler:
    """Online runtime (§4.3): per-stream queues, feedback thresholds, dynamic batching."""

    def __init__(self, ctx: "Context", max_frames_per_tick: int = 65536, snm_slots: int = 65536):
        self.ctx = ctx
        self.handle = ffsva_sched_create(ctx.device, max_frames_per_tick, snm_slots)
        self.cap = max_frames_per_tick + snm_slots
        self._events = np.zeros(self.cap, EVENT_DTYPE)  # reused every tick
        self._n = ctypes.c_int32()
        self._info = TickInfo()

    def push(self, items) -> np.ndarray:
        return ffsva_sched_push(self.handle, Context._frames(items))

    def push_array(self, frames: np.ndarray) -> np.ndarray:
        return ffsva_sched_push_array(self.handle, frames)

    def tick(self, stream=None):
        """One cycle; returns (events copied out of a reused buffer, info dict)."""
        _check(lib().ffsva_sched_tick(self.handle, _stream_handle(stream), self._events.ctypes.data, self.cap,
                                      ctypes.byref(self._n), ctypes.byref(self._info)), "ffsva_sched_tick")
        return self._events[:self._n.value].copy(), self._info.as_dict()

    def depth(self, st: "Stream"):
        return ffsva_sched_depth(self.handle, st.handle)

    def stream_load(self, st: "Stream", reset: bool = False) -> dict:
        """Overload signals of one stream since the last reset (ffsva_sched_stream_load)."""
        out = StreamLoad()
        _check(lib().ffsva_sched_stream_load(self.handle, st.handle, int(reset), ctypes.byref(out)),
               "ffsva_sched_stream_load")
        return out.as_dict()

    def detach(self, st: "Stream") -> bool:
        """True once the stream is detached; False while it still has queued frames / unreported events."""
        r = lib().ffsva_sched_detach(self.handle, st.handle)
        if r == FFSVA_EAGAIN:
            return False
        _check(r, "ffsva_sched_detach")
        return True

    def set_tyolo(self, model, num_tyolo: int = 4, thresh: float = 0.2) -> None:
        """Attach the device's shared T-YOLO stage (a Tyolo, or None to detach): SNM survivors then wait in per-
        stream T-YOLO queues and each tick takes at most num_tyolo frames per stream."""
        _check(lib().ffsva_sched_set_tyolo(self.handle, model.handle if model is not None else None, num_tyolo,
                                           thresh), "ffsva_sched_set_tyolo")

    def set_policy(self, policy: str) -> None:
        """'dynamic' (default), 'feedback' or 'static' (the §5.4 comparison mechanisms)."""
        ffsva_sched_set_policy(self.handle, policy)

    def set_pipeline(self, on: bool) -> bool:
        """Pipelined ticks (ffsva_sched_set_pipeline): tick k harvests cycle k-1's kernels and launches cycle k's
        without waiting. Returns False (mode unchanged) while a cycle is still in flight when switching off."""
        r = lib().ffsva_sched_set_pipeline(self.handle, int(bool(on)))
        if r == FFSVA_EAGAIN:
            return False
        _check(r, "ffsva_sched_set_pipeline")
        return True

    def inspect(self, cap: int = 1 << 16) -> dict:
        """ffsva_sched_inspect: the last launched cycle's frames (stage 0 = SDD admission, 1 = SNM pop) and the
        50x50x3 image each holds in the device slot pool."""
        frames = np.zeros(max(1, cap), dtype=FRAME_DTYPE)
        stage = np.zeros(max(1, cap), np.int32)
        d50 = np.zeros((max(1, cap), 50, 50, 3), np.uint8)
        n = ctypes.c_int32()
        _check(lib().ffsva_sched_inspect(self.handle, frames.ctypes.data, stage.ctypes.data, d50.ctypes.data, cap,
                                         ctypes.byref(n)), "ffsva_sched_inspect")
        k = min(n.value, cap)
        return {"frames": frames[:k], "stage": stage[:k], "d50": d50[:k], "n": n.value}

    def destroy(self) -> None:
        if self.handle:
            ffsva_sched_destroy(self.handle)
            self.handle = None


class PreparedBatch:
    """ffsva_batch_prepare / launch (CUDA graph replay) / fetch."""

    def __init__(self, frames):
        self.n = len(frames)
        self.handle = ffsva_batch_prepare(frames)

    def launch(self, stream=None) -> None:
        ffsva_batch_launch(self.handle, _stream_handle(stream))

    def fetch(self, stream=None, results: bool = True):
        r = ffsva_batch_fetch(self.handle, self.n if results else None, _stream_handle(stream))
        if r is None:
            return None
        return {k: r[k].copy() for k in ("ssd", "sdd_pass", "snm_pass", "snm_class", "logit", "survivor_idx")}

    def device_outputs(self) -> dict:
        return ffsva_batch_device_outputs(self.handle)

    def destroy(self) -> None:
        if self.handle:
            ffsva_batch_destroy(self.handle)
            self.handle = None


# ---------------------------------------------------------------------------------------------- T-YOLO (f1)
TYOLO_GRID = 13


def _bf16_bits_to_f32(u16: np.ndarray) -> np.ndarray:
    return (u16.astype(np.uint32) << 16).view(np.float32)


class Tyolo:
    """The shared T-YOLO stage of a device (NumberofObjects L195; include/ffsva.h)."""

    def __init__(self, ctx: "Context", params: np.ndarray):
        p = np.ascontiguousarray(params, dtype=np.float32)
        h = ctypes.c_void_p()
        _check(lib().ffsva_tyolo_load(ctx.device, p.ctypes.data, p.size, ctypes.byref(h)), "ffsva_tyolo_load")
        self.ctx, self.handle = ctx, h.value

    def run(self, items, target_class: int = 6, thresh: float = 0.2, number_of_objects: int = 1,
            raw: bool = False, stream=None) -> dict:
        """items: (Stream, device pixels, frame_no) as for Context.filter_batch. Returns counts, pass (and raw
        head outputs [n, 13, 13, 125] fp32 when raw=True)."""
        fr = _frames_array(Context._frames(items))
        n = len(items)
        counts = np.zeros(n, np.int32)
        ok = np.zeros(n, np.uint8)
        out = np.zeros((n, TYOLO_GRID, TYOLO_GRID, 125), np.float32) if raw else None
        _check(lib().ffsva_tyolo_run(self.handle, ctypes.addressof(fr), n, target_class, thresh,
                                     number_of_objects, counts.ctypes.data, ok.ctypes.data,
                                     out.ctypes.data if raw else None, _stream_handle(stream)), "ffsva_tyolo_run")
        res = {"counts": counts, "pass": ok}
        if raw:
            res["raw"] = out
        return res

    def layer_output(self, items, layer: int, stream=None) -> np.ndarray:
        """Diagnostic: float32 copy of the bf16 NHWC activation after `layer` (-1 = resized input)."""
        fr = _frames_array(Context._frames(items))
        n = len(items)
        shapes = {-1: (416, 4), 0: (208, 16), 1: (104, 32), 2: (52, 64), 3: (26, 128), 4: (13, 256), 5: (13, 512),
                  6: (13, 1024), 7: (13, 1024)}
        hw, c = shapes[layer]
        out = np.zeros((n, hw, hw, c), np.uint16)
        _check(lib().ffsva_tyolo_layer_output(self.handle, ctypes.addressof(fr), n, layer, out.ctypes.data,
                                              _stream_handle(stream)), "ffsva_tyolo_layer_output")
        return _bf16_bits_to_f32(out)

    def profile(self, items, iters: int = 5, stream=None) -> list:
        """Mean device ms of [resize, layer 1..9] over iters runs (CUDA events on the launching stream)."""
        fr = _frames_array(Context._frames(items))
        ms = (ctypes.c_float * 10)()
        _check(lib().ffsva_tyolo_profile(self.handle, ctypes.addressof(fr), len(items), iters, ms, _stream_handle(stream)),
               "ffsva_tyolo_profile")
        return list(ms)

    def destroy(self) -> None:
        if self.handle:
            _check(lib().ffsva_tyolo_destroy(self.handle), "ffsva_tyolo_destroy")
            self.handle = None
