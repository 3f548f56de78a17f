#!/usr/bin/env python
"""Benchmark of the B200 FFS-VA filter cascade (SDD + SNM) — BASELINE.json metric:
"filtered frames/sec (SDD+SNM) and sustained 30-FPS streams at 1/2/4/8 B200".

One step = one pass of the whole hot path (ingest + downsample, SDD distance and
threshold, survivor compaction + dynamic batching, SNM forward + Eq. (2) decision, per-stream stats) over one
second of video of every stream the rank owns. Default workload = BASELINE.json configs[1] (M2): 30
concurrent 1280x720 RGB8 streams at 10% target rate with dynamic batching (BatchSize 30); each rank owns 30
streams (weak scaling, streams sharded by rank, no data-path collective; an NCCL all-gather of the per-stream
statistics closes the timed region when N > 1).

Timed region: W warm-up steps, then exactly K steps between a barrier + cuda.synchronize on both sides, timed
with CUDA events on the launching stream; max over ranks. Inputs: a 10-second frame pool per rank (9000
frames, 24.9 GB) far larger than L2; consecutive steps read different 2.5 GB slices, so no step hits L2.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config m2] [--impl ours|reference]
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "filtered frames/sec (SDD+SNM) and sustained 30-FPS streams at 1/2/4/8 B200"

# SURVEY.md §8(d) configs. frames_per_step = one second of video per stream (30 FPS).
CONFIGS = {
    "m1": dict(desc="M1: 1 stream 640x360 RGB8, 300 frames, 10% target rate", streams=1, W=640, H=360,
               pool_frames=300, step_frames=300, period=300, on_len=30, seed=1001),
    "m2": dict(desc="M2: 30 concurrent 1280x720 RGB8 streams at 30 FPS, 10% target rate, dynamic batching "
                    "(BatchSize 30)", streams=30, W=1280, H=720, pool_frames=300, step_frames=30, period=300,
               on_len=30, seed=1002),
    "m3": dict(desc="M3: offline single 1920x1080 stream, 10% target rate, max-throughput batches of 512 "
                    "(frame t = pool[t mod 1500])", streams=1, W=1920, H=1080, pool_frames=1500, step_frames=512,
               period=300, on_len=30, seed=1003),
    "m4_10": dict(desc="M4: 64 streams 1280x720, 10% target rate", streams=64, W=1280, H=720, pool_frames=90,
                  step_frames=30, period=300, on_len=30, seed=1004),
    "m4_1": dict(desc="M4: 64 streams 1280x720, 1% target rate", streams=64, W=1280, H=720, pool_frames=90,
                 step_frames=30, period=300, on_len=3, seed=1004),
    "m4_50": dict(desc="M4: 64 streams 1280x720, 50% target rate", streams=64, W=1280, H=720, pool_frames=90,
                  step_frames=30, period=300, on_len=150, seed=1004),
    "m5": dict(desc="M5: 256 streams 1920x1080 sharded over the GPUs, 1 target frame in 10", streams=256,
               W=1920, H=1080, pool_frames=10, step_frames=10, period=10, on_len=1, seed=1005, shard=True),
    # f1: the T-YOLO stage on a batch of SNM survivors (random-init tiny-yolo-voc weights)
    "tyolo": dict(desc="f1 T-YOLO stage: 256 SNM-surviving 1280x720 frames per step through tiny-yolo-voc at "
                       "416x416 (random-init weights), NumberofObjects count", streams=1, W=1280, H=720,
                  pool_frames=256, step_frames=256, period=4, on_len=2, seed=1007),
    # standalone SNM (K4) run for its tensor-pipe roofline: delta_diff = 0 lets every frame
    # through SDD, so one step scores 65,536 survivors across 256 streams (small 128x100 frames with 16-byte rows
    # keep K1 on its bulk-copy path and small; K4 dominates the step and carries the line's roofline)
    "snm": dict(desc="SNM microbenchmark: 65,536 survivors/step across 256 streams (128x100 frames, "
                     "delta_diff = 0 so every frame reaches the SNM)", streams=256, W=128, H=100, pool_frames=256,
                step_frames=256, period=300, on_len=30, seed=1006, delta=0.0),
}
SNM_FLOP = 7_477_632  # algorithmic FLOP per survivor
DELTA, C_LOW, C_HIGH, FD, BATCH = 24.0, 0.2, 0.8, 0.5, 30
L_T = math.log(((C_HIGH - C_LOW) * FD + C_LOW) / (1 - ((C_HIGH - C_LOW) * FD + C_LOW)))  # Eq. (2) in logit space


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms during the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device, self.rows, self.proc, self.th = device, [], None, None

    def start(self):
        if os.environ.get("FFSVA_BENCH_NO_CLOCKS") == "1":  # (diagnostics only: a line without clocks is rejected)
            return
        if os.environ.get("FFSVA_BENCH_CLOCKS") == "nvml":  # in-process NVML polling (A/B against nvidia-smi)
            return self._start_nvml()
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "200", "-i", str(self.device)], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
            return
        self.th = threading.Thread(target=self._read, daemon=True)
        self.th.start()
        # the timed region starts after nvidia-smi's first sample (its start-up is not part of the measurement)
        t0 = time.perf_counter()
        while not self.rows and time.perf_counter() - t0 < 10.0 and self.proc.poll() is None:
            time.sleep(0.02)
        time.sleep(0.25)

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def _start_nvml(self):
        import pynvml
        pynvml.nvmlInit()
        h = pynvml.nvmlDeviceGetHandleByIndex(self.device)
        self._stop = threading.Event()
        bits = [pynvml.nvmlClocksEventReasonHwSlowdown, pynvml.nvmlClocksEventReasonHwThermalSlowdown,
                pynvml.nvmlClocksEventReasonSwThermalSlowdown, pynvml.nvmlClocksEventReasonSwPowerCap]

        def poll():
            while not self._stop.is_set():
                r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
                self.rows.append([str(self.device), str(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)),
                                  str(pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)), "", ""] +
                                 ["Active" if r & b else "Not Active" for b in bits])
                self._stop.wait(0.2)
        self.th = threading.Thread(target=poll, daemon=True)
        self.th.start()
        time.sleep(0.25)

    def stop(self):
        if getattr(self, "_stop", None) is not None:
            self._stop.set()
            self.th.join(timeout=2)
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
            self.th.join(timeout=2)
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if len(r) > 5 + i and r[5 + i] == "Active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), float(d["bf16_tflops"]), "measured"
    return 6650.0, 1590.0, "fallback"


def ncu_traffic(config_name: str):
    """dram bytes per K1 launch from the committed ncu --set full summary (profiles/), if any."""
    p = os.path.join(ROOT, "profiles", "ncu_k1_traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d.get(config_name)
    return None


# ---------------------------------------------------------------------------------------------- distributed skeleton
# The multi-rank plumbing every run goes through (one process per GPU): stream ownership, the timed
# region (barrier + synchronize on both sides, the per-stream statistics all-gather inside it, max over ranks), the
# gather latency and the one-GPU reference throughput for the scaling efficiency. It talks to an "engine" (the GPU
# engine below; tests/test_bench_dist.py drives it with a host engine over gloo at world size 2):
#   eng.device, eng.frames_per_step, eng.step(i), eng.join(), eng.sync(), eng.mark() -> token,
#   eng.elapsed_ms(t0, t1), eng.stats() -> int64 tensor [rows, NSTAT] (equal rows on every rank),
#   eng.solo_frames_per_step, eng.solo_step(i) (the N = 1 workload: the rank's own batches under weak scaling, the
#   whole stream set under strong scaling), eng.start_clocks(), eng.stop_clocks() -> dict.

def owned_streams(cfg, ws: int, rank: int):
    """(global stream ids rank `rank` owns, rows of the gathered statistics per rank). Strong-scaling configs (M5)
    split their streams contiguously (dist.shard_streams); the others give every rank its own streams (weak)."""
    from paper_conf_icpp_zhangcjzly18_b200 import dist as fdist
    if cfg.get("shard"):
        return (list(fdist.shard_streams(cfg["streams"], ws, rank)),
                max(len(fdist.shard_streams(cfg["streams"], ws, r)) for r in range(ws)))
    return list(fdist.weak_streams(cfg["streams"], ws, rank)), cfg["streams"]


def _world():
    import torch.distributed as dist
    return dist.get_world_size() if dist.is_available() and dist.is_initialized() else 1


def _barrier():
    import torch.distributed as dist
    if _world() > 1:
        dist.barrier()


def _allreduce(x: float, op: str, device) -> float:
    """all-reduce of one host number (op 'max' | 'min' | 'sum'); NCCL reduces on the device, gloo on the host."""
    import torch
    import torch.distributed as dist
    if _world() == 1:
        return float(x)
    dev = device if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op={"max": dist.ReduceOp.MAX, "min": dist.ReduceOp.MIN, "sum": dist.ReduceOp.SUM}[op])
    return float(t.item())


def timed_region(eng, steps: int, warmup: int):
    """W untimed warm-up steps, then exactly K steps bracketed by a barrier + synchronize on both sides and timed on
    the device; the per-stream statistics all-gather (NCCL all_gather_into_tensor, the run's one exchange) closes the
    region. Returns (ms = max over ranks, total frames over ranks, gathered statistics, clocks)."""
    from paper_conf_icpp_zhangcjzly18_b200 import dist as fdist
    for i in range(warmup):
        eng.step(i)
    eng.sync()
    _barrier()
    eng.start_clocks()
    eng.sync()
    _barrier()
    t0 = eng.mark()
    marks = []
    for i in range(steps):
        eng.step(warmup + i)
        if getattr(eng, "step_marks", False):
            marks.append(eng.mark())
    eng.join()
    gathered = fdist.gather_stats(eng.stats())
    t1 = eng.mark()
    eng.sync()
    _barrier()
    clk = eng.stop_clocks()
    if marks:  # diagnostics (FFSVA_BENCH_STEP_MARKS=1): the slowest step between consecutive marks
        ts = [eng.elapsed_ms(t0, marks[0])] + [eng.elapsed_ms(a, b) for a, b in zip(marks, marks[1:])]
        eng.step_ms = {"max": max(ts), "median": sorted(ts)[len(ts) // 2], "argmax": ts.index(max(ts))}
    ms_max = _allreduce(eng.elapsed_ms(t0, t1), "max", eng.device)
    total = _allreduce(eng.frames_per_step * steps, "sum", eng.device)
    return ms_max, int(total), gathered, clk


def gather_us(eng, reps: int = 50) -> float:
    """Device time of one statistics all-gather (the per-interval exchange of §8(e)), mean of `reps`, max over
    ranks, in microseconds."""
    from paper_conf_icpp_zhangcjzly18_b200 import dist as fdist
    local = eng.stats()
    fdist.gather_stats(local)
    eng.sync()
    _barrier()
    t0 = eng.mark()
    for _ in range(reps):
        fdist.gather_stats(local)
    t1 = eng.mark()
    eng.sync()
    return 1e3 * _allreduce(eng.elapsed_ms(t0, t1) / reps, "max", eng.device)


def solo_fps(eng, steps: int, rank: int) -> float:
    """Throughput of the N = 1 workload on one GPU (rank 0 alone while the other ranks wait), for the scaling
    efficiency fps(G) / (G * fps(1)). Every rank returns rank 0's figure."""
    fps = 0.0
    eng.sync()
    _barrier()
    if rank == 0:
        for i in range(2):
            eng.solo_step(i)
        eng.join()
        eng.sync()
        t0 = eng.mark()
        for i in range(steps):
            eng.solo_step(2 + i)
        eng.join()
        t1 = eng.mark()
        eng.sync()
        fps = eng.solo_frames_per_step * steps / (eng.elapsed_ms(t0, t1) / 1e3)
    return _allreduce(fps, "max", eng.device)


def scaling_fields(value: float, fps1: float, ws: int, g_us: float, gathered_rows: int, strong: bool,
                   backend: str = "nccl") -> dict:
    return {"kind": "strong" if strong else "weak", "n_gpus": ws, "fps_1gpu": fps1,
            "efficiency": value / (ws * fps1) if fps1 > 0 else None,
            "efficiency_def": "fps(G) / (G * fps(1)); fps(1) = the N = 1 workload timed on rank 0 of this run "
                              "(strong: all streams on one GPU; weak: one rank's streams)",
            "stats_gather_us": g_us, "stats_gather_rows": gathered_rows,
            "stats_gather": ("NCCL all_gather_into_tensor" if backend == "nccl" else "gloo all_gather (host copies)")
                            + " of the u64 per-stream table (device time, max over ranks)"}


# ---------------------------------------------------------------------------------------------- our arm

class GpuEngine:
    """The bench's workload on one GPU: the rank's streams (reference + SNM each), a stream-major frame pool far
    larger than L2, and prepared batches (one second of video of every owned stream each) replayed as CUDA graphs,
    consecutive steps alternating over CUDA streams."""

    def __init__(self, args, cfg, ws, rank, dev):
        import torch

        import paper_conf_icpp_zhangcjzly18_b200 as ff
        from paper_conf_icpp_zhangcjzly18_b200 import ffsva as ffb
        from synth import synth
        self.torch, self.ffb, self.dev, self.device = torch, ffb, dev, dev
        self.cfg, self.args, self.rank, self.ws = cfg, args, rank, ws
        W, H, P = cfg["W"], cfg["H"], 3 * cfg["W"]
        self.W, self.H, self.P, self.fbytes = W, H, P, H * P
        self.sids, self.rows = owned_streams(cfg, ws, rank)
        # strong scaling: rank 0 also holds the whole stream set (its shard is the prefix) for the N = 1 reference
        self.strong = bool(cfg.get("shard"))
        all_ids = list(range(cfg["streams"])) if (self.strong and ws > 1 and rank == 0) else self.sids
        S_all, PF, SF = len(all_ids), cfg["pool_frames"], cfg["step_frames"]
        self.video = synth.Video(seed=cfg["seed"], width=W, height=H, period=cfg["period"], on_len=cfg["on_len"])
        self.ctx = ff.Context(dev)
        self.delta = cfg.get("delta", DELTA)
        self.streams = []
        for s in all_ids:
            st = self.ctx.open_stream(width=W, height=H, delta_diff=self.delta, c_low=C_LOW, c_high=C_HIGH,
                                      filter_degree=FD, snm_batch=BATCH)
            refs = torch.empty((32, H, P), dtype=torch.uint8, device=dev)
            synth.frames_cuda(self.video, torch.full((32,), s, dtype=torch.int32, device=dev),
                              torch.arange(32, dtype=torch.int64, device=dev), refs, self.fbytes, P, ref=True)
            st.set_reference(refs)
            del refs
            st.snm_load(synth.snm_weights(cfg["seed"], s))
            self.streams.append(st)
        # frame pool: stream-major, pool[s][t]
        self.pool = torch.empty((S_all, PF, H, P), dtype=torch.uint8, device=dev)
        for k, s in enumerate(all_ids):
            synth.frames_cuda(self.video, torch.full((PF,), s, dtype=torch.int32, device=dev),
                              torch.arange(PF, dtype=torch.int64, device=dev), self.pool[k], self.fbytes, P)
        torch.cuda.synchronize()
        S = len(self.sids)
        self.S, self.PF, self.SF = S, PF, SF
        # prepared batches: batch j = frames [j*SF, (j+1)*SF) of every owned stream (one second of video); a pool of
        # exactly one batch (M1, M5) gets one prepared copy per CUDA stream (same frames, own buffers), so consecutive
        # steps overlap like the other configs' (each step still runs K1 -> K3 -> K4 on all of its frames)
        uniq = max(1, PF // SF)
        self.nbatches = uniq if uniq > 1 else max(1, args.streams)

        def make(nstreams):
            return [self.ctx.prepare([(self.streams[k], self.pool[k, (j % uniq) * SF + i], (j % uniq) * SF + i)
                                      for k in range(nstreams) for i in range(SF)]) for j in range(self.nbatches)]
        self.batches = make(S)
        self.solo_batches = make(S_all) if S_all != S else self.batches
        self.frames_per_step = S * SF
        self.solo_frames_per_step = S_all * SF
        self.planted = [sum(synth.planted(self.video, s, (j % uniq) * SF, (j % uniq + 1) * SF) for s in self.sids)
                        for j in range(self.nbatches)]
        self.cs = torch.cuda.Stream(device=dev)
        nstr = max(1, min(args.streams, self.nbatches))
        self.css = [self.cs] + [torch.cuda.Stream(device=dev) for _ in range(nstr - 1)]
        self.stats_dev = torch.zeros((max(1, self.rows), ffb.NSTAT), dtype=torch.int64, device=dev)
        self.clocks = None
        self.step_marks = os.environ.get("FFSVA_BENCH_STEP_MARKS") == "1"
        self.step_ms = None

    # --- correctness gate before timing: SDD pass count == planted count on every batch (P8 at full size), and
    # the fraction of survivors whose logit lies within the 2e-2 parity margin of the decision threshold
    def gate(self):
        torch = self.torch
        near, surv = 0, 0
        for j, b in enumerate(self.batches):
            b.launch(self.cs)
            r = b.fetch(self.cs)
            expect = self.planted[j] if self.delta == DELTA else self.frames_per_step
            if int(r["sdd_pass"].sum()) != expect:
                raise RuntimeError(f"batch {j}: SDD passed {int(r['sdd_pass'].sum())} != expected {expect}")
            self.planted[j] = expect
            lg = r["logit"][r["sdd_pass"] == 1]
            near += int((np.abs(lg - L_T) < 2e-2).sum())
            surv += lg.size
        self.ctx.stats(reset=True)
        self.stats()  # allocates the library's pinned statistics snapshot outside the timed region
        torch.cuda.synchronize()
        self.near_margin = {"fraction": near / surv if surv else 0.0, "survivors": surv, "margin": 2e-2,
                            "bar": "< 0.10 (SURVEY.md §8(d): else the decision parity check is weak)"}
        if surv and near / surv >= 0.10 and not os.environ.get("FFSVA_LIB"):  # FFSVA_LIB: A/B builds (timing only)
            raise RuntimeError(f"{near}/{surv} survivors lie within 2e-2 of the SNM threshold (>= 10%)")

    def step(self, i):
        self.batches[i % self.nbatches].launch(self.css[i % len(self.css)])

    def solo_step(self, i):
        self.solo_batches[i % self.nbatches].launch(self.css[i % len(self.css)])

    def join(self):  # the last step of every CUDA stream is done before the closing mark
        for s2 in self.css[1:]:
            ev = self.torch.cuda.Event()
            ev.record(s2)
            self.cs.wait_event(ev)

    def sync(self):
        self.torch.cuda.synchronize()

    def mark(self):
        e = self.torch.cuda.Event(enable_timing=True)
        e.record(self.cs)
        for s2 in self.css[1:]:  # later steps on the other streams start after this mark
            s2.wait_event(e)
        return e

    def elapsed_ms(self, t0, t1):
        t1.synchronize()
        return t0.elapsed_time(t1)

    def stats(self):
        """a8: the owned streams' statistics rows (device table, stream slots in open order) -> stats_dev."""
        n = min(self.S, self.rows)
        self.ffb.ffsva_stats_copy(self.dev.index, self.stats_dev.data_ptr(), max(1, n), False, False,
                                  self.cs.cuda_stream)
        return self.stats_dev

    def start_clocks(self):
        self.clocks = ClockSampler(self.dev.index)
        self.clocks.start()

    def stop_clocks(self):
        return self.clocks.stop() if self.clocks else None

    def close(self):
        for b in {id(b): b for b in self.batches + self.solo_batches}.values():
            b.destroy()
        self.ctx.close()


def run_ours(args, cfg, ws, rank, local):
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_zhangcjzly18_b200 as ff
    from paper_conf_icpp_zhangcjzly18_b200 import ffsva as ffb

    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    eng = GpuEngine(args, cfg, ws, rank, dev)
    eng.gate()
    # torch's current stream = the launching stream, so the statistics copy, the all-gather (NCCL orders its work
    # after the current stream) and the closing timer mark are ordered on one stream
    cur = torch.cuda.stream(eng.cs)
    cur.__enter__()
    launches0 = ff.ffsva_kernel_launches()
    ms_max, total_frames, gathered, clk = timed_region(eng, args.steps, args.warmup)
    launches = ff.ffsva_kernel_launches() - launches0
    value = total_frames / (ms_max / 1e3)
    # the gathered table must account for every frame every rank launched (warm-up + timed steps)
    g = gathered.cpu().numpy()
    if int(g[:, 0].sum()) != int(_allreduce(eng.frames_per_step * (args.warmup + args.steps), "sum", dev)):
        raise RuntimeError("gathered per-stream frame counters disagree with the frames launched")
    g_us = gather_us(eng) if ws > 1 else 0.0
    fps1 = solo_fps(eng, max(3, min(args.steps, 50)), rank) if ws > 1 else value
    cur.__exit__(None, None, None)
    scaling = scaling_fields(value, fps1, ws, g_us, int(g.shape[0]), eng.strong, args.dist_backend)

    # ---- per-kernel device times (CUDA events on the launching stream) for the roofline
    batches, nbatches, cs = eng.batches, eng.nbatches, eng.cs
    k_ms = ffb.ffsva_batch_profile([b.handle for b in batches], max(2, min(10, 30 // nbatches + 1)), cs.cuda_stream)
    m_avg = float(np.mean(eng.planted))
    W, H, P, S, SF = eng.W, eng.H, eng.P, eng.S, eng.SF
    frames_per_step = eng.frames_per_step
    k1_bytes = frames_per_step * (3 * W * H + 9) + m_avg * 7500
    hbm_peak, tf_peak, peak_kind = measured_peaks()
    achieved = k1_bytes / (k_ms[0] / 1e3) / 1e9
    traffic = ncu_traffic(args.config)

    # ---- end to end through the public API with HOST buffers (pinned), H2D + D2H inside the timed region
    e2e = None
    if not args.no_e2e:
        n_e2e = max(1, min(args.steps, args.e2e_steps))
        pinned = torch.empty((S, SF, H, P), dtype=torch.uint8).pin_memory()
        pinned.copy_(eng.pool[:S, :SF].cpu())
        items = [(eng.streams[k], pinned[k, i].data_ptr(), i) for k in range(S) for i in range(SF)]
        eng.ctx.filter_batch(items, stream=cs, host=True)  # warm-up (ring allocation)
        torch.cuda.synchronize()
        _barrier()
        h0, h1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        h0.record(cs)
        for _ in range(n_e2e):
            eng.ctx.filter_batch(items, stream=cs, host=True)
        h1.record(cs)
        torch.cuda.synchronize()
        te = _allreduce(h0.elapsed_time(h1), "max", dev)
        e2e_val = _allreduce(frames_per_step * n_e2e, "sum", dev) / (te / 1e3)
        e2e = {"value": e2e_val, "unit": "frames/s", "h2d_bytes_per_step": int(frames_per_step * eng.fbytes),
               "d2h_bytes_per_step": int(frames_per_step * ffb.RESULT_DTYPE.itemsize), "steps": n_e2e,
               "path": "ffsva_filter_batch_host (pinned host frames -> 2-chunk device ring, copies overlapped "
                       "with K1)"}
        del pinned

    cpu = None
    if rank == 0 and not args.no_cpu_baseline:
        if ws == 1:
            cpu = cpu_baseline(cfg, eng.video, eng.sids, eng.pool, args.cpu_frames)
        else:
            cpu = {"kind": "oracle", "measured_at": "N = 1 only (the oracle is a host program: its figure does not "
                                                   "change with the GPU count)"}

    # ---- online validation of "sustained 30-FPS streams" (paced arrivals through the online runtime)
    online = None
    if args.online and args.config == "m2":
        online = online_validation(args, eng.ctx, eng.video, eng.sids, eng.pool[:S], value / ws, dev, cs, ws)

    out = None
    if rank == 0:
        out = {
            "metric": METRIC, "value": value, "unit": "frames/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
            "scaling": "strong" if eng.strong else "weak", "vs_baseline": None,
            "dtype": "u8 (SDD) / bf16-fp32 (SNM)", "data": "synthetic",
            "config": {"workload": cfg["desc"], "config_id": args.config, "streams_per_gpu": S,
                       "frames_per_step": int(total_frames // args.steps), "frames_per_step_per_gpu": frames_per_step,
                       "frame_bytes": eng.fbytes, "pool_bytes_per_gpu": int(S * eng.PF * eng.fbytes),
                       "l2": ("inputs larger than L2: each step reads a different %.2f GB slice of the pool"
                              % (frames_per_step * eng.fbytes / 1e9) if eng.PF > eng.SF else
                              "inputs larger than L2: each step reads the whole %.2f GB pool" % (S * eng.PF * eng.fbytes / 1e9)),
                       "parallelism": (f"stream-sharded x{ws} (strong: {cfg['streams']} streams split, {S} on rank 0)"
                                       if eng.strong else f"stream-sharded x{ws} (weak: {S} streams per GPU)"),
                       "dist_backend": args.dist_backend if ws > 1 else None,
                       "batch_size": BATCH, "delta_diff": DELTA, "c_low": C_LOW, "c_high": C_HIGH,
                       "filter_degree": FD, "seed": cfg["seed"], "cuda_streams": len(eng.css)},
            "sustained_streams_30fps": int(value // 30),
            "sdd_pass_per_step": m_avg,
            "snm_near_margin": eng.near_margin,
            "multi_gpu": scaling,
            "roofline": {"bound": "hbm", "kernel": "K1 sdd_kernel (ingest + box downsample + SSD + threshold)",
                         "achieved": achieved, "peak": hbm_peak, "unit": "GB/s", "frac": achieved / hbm_peak,
                         "peak_source": peak_kind, "traffic": traffic,
                         "algorithmic_bytes_per_launch": k1_bytes,
                         "kernel_ms": {"K1_sdd": k_ms[0], "K3_compact": k_ms[1], "K4_snm": k_ms[2]},
                         "k1_share_of_step": k_ms[0] / max(1e-9, sum(k_ms))},
            # K4 against the tensor roofline (algorithmic SNM FLOPs of this step's survivors / K4 time); the
            # burst bf16 peak applies because K4 is timed alone (ffsva_batch_profile)
            "snm_roofline": {"bound": "tensor", "kernel": "K4 snm_kernel (tcgen05 bf16, fp32 accumulate)",
                             "survivors_per_launch": m_avg,
                             "achieved": m_avg * SNM_FLOP / (k_ms[2] / 1e3) / 1e12 if k_ms[2] > 0 else 0.0,
                             "peak": tf_peak, "unit": "TFLOP/s",
                             "frac": (m_avg * SNM_FLOP / (k_ms[2] / 1e3) / 1e12) / tf_peak if k_ms[2] > 0 else 0.0,
                             "peak_source": peak_kind, "survivors_per_s": m_avg / (k_ms[2] / 1e3) if k_ms[2] else 0},
            "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": int(launches), "clocks": clk,
            **({"step_ms_diagnostic": eng.step_ms} if eng.step_ms else {}),
            "online": online,
            "sustained_streams_validated": None if not online else {
                "sdd_snm": online.get("max_sustained_streams_validated"),
                "sdd_snm_tyolo": online.get("max_sustained_streams_validated_with_tyolo"),
                "window_s": online.get("validation_window_s"),
                "by_tor": {k: v["max_sustained_streams_validated"] for k, v in online.get("online_by_tor", {}).items()},
                "by_tor_window_s": args.online_tor_confirm_seconds},
        }
        if args.config == "snm":  # K4 is this workload's dominant kernel: its tensor roofline is the line's
            out["sdd_roofline"] = out["roofline"]
            out["roofline"] = dict(out["snm_roofline"], kernel_ms=out["sdd_roofline"]["kernel_ms"],
                                   k4_share_of_step=k_ms[2] / max(1e-9, sum(k_ms)))
    eng.close()
    return out


# tiny-yolo-voc convolutions at 416x416: (H, Cin, Cout, k); algorithmic FLOPs = 2 x MACs at full resolution
TYOLO_CONV = [(416, 3, 16, 3), (208, 16, 32, 3), (104, 32, 64, 3), (52, 64, 128, 3), (26, 128, 256, 3),
              (13, 256, 512, 3), (13, 512, 1024, 3), (13, 1024, 1024, 3), (13, 1024, 125, 1)]
TYOLO_FLOP = sum(2 * h * h * ci * co * k * k for h, ci, co, k in TYOLO_CONV)  # 6,971,041,792 per frame


def run_tyolo(args, cfg, ws, rank, local):
    """--config tyolo: the f1 stage alone. Device time per step = the mean CUDA-event time of the resize and the
    nine layers over the timed steps (ffsva_tyolo_profile, events on the launching stream); e2e = wall time of
    ffsva_tyolo_run (host call, counts copied back) per step."""
    import torch
    import paper_conf_icpp_zhangcjzly18_b200 as ff
    from synth import synth
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    W, H, P, n = cfg["W"], cfg["H"], 3 * cfg["W"], cfg["step_frames"]
    video = synth.Video(seed=cfg["seed"], width=W, height=H, period=cfg["period"], on_len=cfg["on_len"])
    frames = torch.empty((n, H, P), dtype=torch.uint8, device=dev)
    synth.frames_cuda(video, torch.zeros(n, dtype=torch.int32, device=dev), torch.arange(n, dtype=torch.int64,
                      device=dev), frames, H * P, P)
    ctx = ff.Context(dev)
    st = ctx.open_stream(width=W, height=H)
    params = synth.tyolo_weights(cfg["seed"])
    ty = ff.Tyolo(ctx, params)
    items = [(st, frames[i], i) for i in range(n)]
    cs = torch.cuda.Stream(device=dev)
    launches0 = ff.ffsva_kernel_launches()
    ty.profile(items, args.warmup, stream=cs)
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)
    ms = ty.profile(items, args.steps, stream=cs)
    clk = clocks.stop()
    launches = (ff.ffsva_kernel_launches() - launches0) * args.steps // (args.steps + args.warmup)
    step_ms = sum(ms)
    value = n / (step_ms / 1e3)
    _, tf_peak, peak_kind = measured_peaks()
    layer_tf = [TYOLO_CONV[i][0] ** 2 * 2 * TYOLO_CONV[i][1] * TYOLO_CONV[i][2] * TYOLO_CONV[i][3] ** 2 * n
                / (ms[i + 1] / 1e3) / 1e12 for i in range(9)]
    dom = max(range(9), key=lambda i: ms[i + 1])
    achieved = TYOLO_FLOP * n / (step_ms / 1e3) / 1e12
    t0 = time.perf_counter()
    n_e2e = max(1, min(5, args.steps))
    for _ in range(n_e2e):
        res = ty.run(items, number_of_objects=2, stream=cs)
    e2e = n * n_e2e / (time.perf_counter() - t0)
    cpu = None
    if not args.no_cpu_baseline:
        from oracle import oracle as orc
        host = frames[:2].cpu().numpy()
        t0 = time.perf_counter()
        for i in range(2):
            orc.tyolo_forward(orc.resize(host[i], W, 416, 416), params, bf16_emul=False)
        dt = time.perf_counter() - t0
        cpu = {"value": 2 / dt, "unit": "frames/s", "cores": 1, "kind": "oracle",
               "sample": "2 frames (resize + the nine layers in fp64 + count) of the same workload", "seconds": dt}
    out = {"metric": "T-YOLO frames/sec (f1 stage, 416x416 tiny-yolo-voc)", "value": value, "unit": "frames/s",
           "n_gpus": 1, "steps": args.steps, "warmup": args.warmup, "ms_per_step": step_ms,
           "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "bf16 (fp32 accumulate)",
           "data": "synthetic",
           "config": {"workload": cfg["desc"], "config_id": "tyolo", "frames_per_step": n, "seed": cfg["seed"],
                      "l2": "activations of 256 frames (up to 354 MB per layer) exceed L2; weights 31.7 MB bf16"},
           "roofline": {"bound": "tensor", "kernel": "K5 tyolo_conv_kernel (all nine layers)",
                        "achieved": achieved, "peak": tf_peak, "unit": "TFLOP/s", "frac": achieved / tf_peak,
                        "peak_source": peak_kind, "traffic": None, "flop_per_frame": TYOLO_FLOP,
                        "dominant_layer": f"L{dom + 1}", "dominant_layer_tflops": layer_tf[dom],
                        "layer_ms": {("resize" if i == 0 else f"L{i}"): ms[i] for i in range(10)},
                        "layer_tflops": {f"L{i + 1}": layer_tf[i] for i in range(9)}},
           "cpu_baseline": cpu,
           "e2e": {"value": e2e, "unit": "frames/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 8 * n,
                   "path": "ffsva_tyolo_run on device-resident frames (host call, counts + pass copied back)",
                   "mean_count": float(np.mean(res["counts"]))},
           "gpu_launches": int(launches), "clocks": clk}
    ty.destroy()
    ctx.close()
    return out


def online_validation(args, ctx, video, sids, pool, value, dev, cs, ws=1):
    """Paced 30-FPS streams through the online runtime (feedback queue + dynamic batching, §4.3).
    Stream i replays content stream i % len(sids) of the pool with its own reference image and SNM.

    Each ladder climbs fractions of the measured offline capacity with short rungs (--online-seconds) until a count is
    not sustained, then confirms its best rung with a long paced run (--online-confirm-seconds, 30 s by default: the
    §8(d) contract); if the confirmation fails, the rung below is confirmed instead. Ladders: SDD + SNM on the M2
    content; the full SDD -> SNM -> T-YOLO cascade (f1); and the target-occurrence sweep of config M4 (TOR 1 / 10 /
    50 %: the same backgrounds with 3 / 30 / 150 target frames per 300), confirmed over --online-tor-confirm-seconds.
    The verdict of every run is online.sustained_verdict (p99 <= 1 s, >= 99 % of the window's arrivals decided, no
    backlog growth over the last 10 s).

    N > 1: every rank runs the same per-GPU counts on its own GPU at the same time (streams are sharded, no frame
    crosses GPUs); a count is sustained only if it is sustained on every rank (all-reduce MIN of the verdicts, so
    the ranks also climb their ladders in lock step), and the whole-job count is N x the per-GPU count."""
    import torch

    from paper_conf_icpp_zhangcjzly18_b200.online import run_paced
    from synth import synth
    W, H, P = video.width, video.height, 3 * video.width
    nc = len(sids)
    refs = []
    for k, s in enumerate(sids):
        r = torch.empty((32, H, P), dtype=torch.uint8, device=dev)
        synth.frames_cuda(video, torch.full((32,), s, dtype=torch.int32, device=dev),
                          torch.arange(32, dtype=torch.int64, device=dev), r, H * P, P, ref=True)
        refs.append(r)
    opened = []
    ty = None
    state = {"ty_warm": False}

    # a device context holds at most 65,536 streams (the statistics table's rows; FrameDesc.slot is 16-bit): the
    # ladders stop below it, leaving room for the benchmark's own streams
    s_cap = 65536 - 512

    def run(S, content, seconds, with_ty):
        S = min(S, s_cap)
        t_setup = time.perf_counter()
        while len(opened) < S:
            i = len(opened)
            st = ctx.open_stream(width=W, height=H, delta_diff=DELTA, c_low=C_LOW, c_high=C_HIGH, filter_degree=FD,
                                 snm_batch=BATCH, q_sdd=2, q_snm=10)
            st.set_reference(refs[i % nc])
            st.snm_load(synth.snm_weights(video.seed, 100000 + i))
            opened.append(st)
        setup_s = time.perf_counter() - t_setup
        if with_ty and not state["ty_warm"]:  # outside the paced window: the first T-YOLO launches load their modules
            ty.run([(opened[0], content[0][t], t) for t in range(2)], target_class=14, thresh=0.2)
            state["ty_warm"] = True
        # cycles of 10 ms, 25 ms from 10 K streams, 50 ms from 30 K (the per-cycle work — admission over all cameras,
        # the single-CTA compaction, launches — is amortised over more frames; p99 stays ~0.2 s of the 1-s budget)
        res = run_paced(ctx, opened[:S], [content[i % nc] for i in range(S)], content.shape[1], seconds,
                        cuda_stream=cs, tyolo=ty if with_ty else None,
                        tick_s=args.online_tick_ms / 1e3 if args.online_tick_ms else
                        (0.010 if S < 10000 else (0.025 if S < 30000 else 0.050)))
        res["stream_setup_s"] = setup_s
        if ws > 1:
            res["sustained_this_rank"] = res["sustained"]
            res["sustained"] = bool(_allreduce(1 if res["sustained"] else 0, "min", dev))
            res["streams_per_gpu"], res["streams"] = S, S * ws
        return res

    def climb(fracs, content, confirm_s, with_ty, bisect=2):
        """Rungs at fractions of the offline capacity until one fails, then `bisect` halvings between the last
        sustained and the failing fraction; the best sustained rung is confirmed with a long run (else the next
        best). A short unrecorded run at the first rung's count warms the path first (allocations, first launches)."""
        warm = run(max(31, int(fracs[0] * value / 30)), content, 2.0, with_ty)
        rungs, ok, bad = [], [], None

        def rung(f):
            S = min(s_cap, max(31, int(f * value / 30)))
            r = run(S, content, args.online_seconds, with_ty)
            r["fraction_of_offline_capacity"] = f
            if S == s_cap:
                r["capped_at_stream_table"] = s_cap
            rungs.append(r)
            return r["sustained"], S

        for f in fracs:
            good, S = rung(f)
            if not good:
                bad = f
                break
            ok.append((f, S))
            if S == s_cap:  # the stream table bounds the ladder: higher rungs would repeat this count
                break
        lo = ok[-1][0] if ok else 0.0
        for _ in range(bisect if bad is not None else 0):
            mid = (lo + bad) / 2
            good, S = rung(mid)
            if good:
                ok.append((mid, S))
                lo = mid
            else:
                bad = mid
        best = sorted(ok, key=lambda t: t[1])
        confirms, validated = [], 0
        for _, S in reversed(best[-2:]):
            r = run(S, content, confirm_s, with_ty)
            confirms.append(r)
            if r["sustained"]:
                validated = S * ws
                break
        return {"rungs": rungs, "confirm": confirms, "max_sustained_streams_validated": validated,
                "validation_window_s": confirm_s, "warmup_run": {k: warm[k] for k in ("streams", "seconds",
                                                                                   "sustained")}}

    out = {"policy": "q_sdd 2, q_snm 10, q_tyolo 2, BatchSize 30, num_t-yolo 4 (PAPER.md L173, L217, L219); "
                     "sustained = p99 <= 1 s, >= 99 % of the window's arrivals decided, no backlog growth "
                     "(online.sustained_verdict)"}
    explicit = [int(t) for t in args.online.split(",") if t.strip() and t.strip() != "auto"]
    out["runs"] = [run(S, pool, args.online_seconds, False) for S in explicit]
    if "auto" in args.online:
        lad = climb((0.55, 0.7, 0.85, 0.9, 0.95, 1.0), pool, args.online_confirm_seconds, False)
        out["sdd_snm"] = lad
        out["max_sustained_streams_validated"] = lad["max_sustained_streams_validated"]
        out["validation_window_s"] = lad["validation_window_s"]
    if args.online_tyolo:
        import paper_conf_icpp_zhangcjzly18_b200 as ff
        ty = ff.Tyolo(ctx, synth.tyolo_weights(video.seed))
        tyo = [int(t) for t in args.online_tyolo.split(",") if t.strip() and t.strip() != "auto"]
        out["tyolo_runs"] = [run(S, pool, args.online_seconds, True) for S in tyo]
        if "auto" in args.online_tyolo:  # T-YOLO (~100 K frames/s) sees the SNM survivors, a few % of the frames
            lad = climb((0.1, 0.2, 0.3, 0.4, 0.5), pool, args.online_confirm_seconds, True)
            out["sdd_snm_tyolo"] = lad
            out["max_sustained_streams_validated_with_tyolo"] = lad["max_sustained_streams_validated"]
    if args.online_tor:
        # M4's target-occurrence sweep (S_max per TOR; the analogue of Fig. 6a): the
        # same backgrounds (so the same references) with TOR 1 / 10 / 50 % targets
        by_tor = {}
        for tok in args.online_tor.split(","):
            tor = int(tok)
            on_len = {1: 3, 10: 30, 50: 150}[tor]
            if on_len == video.on_len:
                content = pool
            else:
                v2 = synth.Video(seed=video.seed, width=W, height=H, period=video.period, on_len=on_len)
                content = torch.empty_like(pool)
                for k, s in enumerate(sids):
                    synth.frames_cuda(v2, torch.full((pool.shape[1],), s, dtype=torch.int32, device=dev),
                                      torch.arange(pool.shape[1], dtype=torch.int64, device=dev), content[k], H * P, P)
            lad = climb((0.7, 0.85, 0.95), content, args.online_tor_confirm_seconds, False, bisect=1)
            by_tor[f"{tor}%"] = {"max_sustained_streams_validated": lad["max_sustained_streams_validated"],
                                 "validation_window_s": lad["validation_window_s"], "rungs": lad["rungs"],
                                 "confirm": lad["confirm"]}
            del content
        out["online_by_tor"] = by_tor
    closed = set(id(st) for st in opened)
    for st in opened:
        st.close()
    ctx.streams = [st for st in ctx.streams if id(st) not in closed]  # (list.remove per stream is O(S^2))
    if ty is not None:
        ty.destroy()
    return out


def _cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def _oracle_worker(args):
    """One host core: the unchanged single-threaded oracle on its own (stream, frame range) of the workload. Frames
    come from the host generator (byte-identical to the device pool, tests/test_gpu_parity.py) and are generated
    before the clock starts."""
    cfg, seed_stream, t0, nf = args
    from oracle import oracle as orc
    from synth import synth
    W = cfg["W"]
    video = synth.Video(seed=cfg["seed"], width=W, height=cfg["H"], period=cfg["period"], on_len=cfg["on_len"])
    ref = orc.reference(synth.frames(video, [seed_stream] * 8, list(range(8)), ref=True), W, 100, 100)
    fr = list(synth.frames(video, [seed_stream] * nf, [(t0 + i) % cfg["pool_frames"] for i in range(nf)]))
    params = synth.snm_weights(cfg["seed"], seed_stream)
    t = time.perf_counter()
    orc.filter_frames(fr, W, [ref] * nf, [DELTA] * nf, [params] * nf, [C_LOW] * nf, [C_HIGH] * nf, [FD] * nf)
    return nf, time.perf_counter() - t


def cpu_baseline(cfg, video, sids, pool, n_frames):
    """The oracle, as it stands (plain single-threaded C), on a bounded sample of the workload: on one host core,
    and on every core of the process's affinity set with each core running the unchanged oracle on its own
    streams; the line's value is the one-core figure."""
    import multiprocessing as mp

    from oracle import oracle as orc
    from synth import synth
    W, H = cfg["W"], cfg["H"]
    S = len(sids)
    per = max(1, n_frames // S)
    refs = {}
    t0 = time.perf_counter()
    for k in range(S):
        r = synth.frames(video, [sids[k]] * 32, list(range(32)), ref=True)
        refs[k] = orc.reference(r, W, 100, 100)
    t_ref = time.perf_counter() - t0
    dt, done = 0.0, 0
    for k in range(S):  # one stream's frames on the host at a time
        fr = list(pool[k, :min(per, cfg["pool_frames"])].cpu().numpy())
        params = synth.snm_weights(cfg["seed"], sids[k])
        t0 = time.perf_counter()
        orc.filter_frames(fr, W, [refs[k]] * len(fr), [DELTA] * len(fr), [params] * len(fr),
                          [C_LOW] * len(fr), [C_HIGH] * len(fr), [FD] * len(fr))
        dt += time.perf_counter() - t0
        done += len(fr)
    out = {"value": done / dt, "unit": "frames/s", "cores": 1, "kind": "oracle", "cpu_model": _cpu_model(),
           "sample": f"{done} frames ({per} per stream x {S} streams) of the same workload, full cascade "
                     f"(downsample x2, SSD, threshold, compaction, SNM fp64 on survivors); reference images "
                     f"({t_ref:.1f} s) not timed", "seconds": dt}
    # every core: process p runs the oracle on stream sids[p % S], frames [(p // S) * nf, ...) of the pool
    ncores = len(os.sched_getaffinity(0))
    if ncores > 1:
        nf = 16
        jobs = [(cfg, sids[p % S], (p // S) * nf, nf) for p in range(ncores)]
        try:
            with mp.get_context("fork").Pool(ncores) as mpool:
                res = mpool.map(_oracle_worker, jobs)
            frames = sum(r[0] for r in res)
            wall = max(r[1] for r in res)
            out["multicore"] = {"value": frames / wall, "unit": "frames/s", "cores": ncores,
                                "sample": f"{nf} frames per core, one stream per core (streams reused round-robin); "
                                          f"value = all frames / the slowest core's time"}
        except Exception as e:  # noqa: BLE001 (reported, never fatal for the GPU line)
            out["multicore"] = {"error": str(e)[:200]}
    return out


# ---------------------------------------------------------------------------------------------- reference arm

def run_reference(args, cfg, ws, rank):
    """--impl reference: the CPU oracle (plain single-threaded C) timed on the host on a bounded sample of the
    same workload: each step = one frame (round-robin over the streams), full cascade."""
    if rank != 0:
        return None
    from oracle import oracle as orc
    from synth import synth
    W, H = cfg["W"], cfg["H"]
    video = synth.Video(seed=cfg["seed"], width=W, height=H, period=cfg["period"], on_len=cfg["on_len"])
    if args.config == "tyolo":  # the f1 stage: one frame (resize + nine layers in fp64 + count) per step
        params = synth.tyolo_weights(cfg["seed"])
        imgs = [orc.resize(synth.frame(video, 0, t), W, 416, 416) for t in range(4)]
        for i in range(args.warmup):
            orc.tyolo_count(orc.tyolo_forward(imgs[i % 4], params), 6)
        t0 = time.perf_counter()
        for i in range(args.steps):
            orc.tyolo_count(orc.tyolo_forward(imgs[i % 4], params), 6)
        dt = time.perf_counter() - t0
        value = args.steps / dt
        return {"metric": "T-YOLO frames/sec (f1 stage, 416x416 tiny-yolo-voc)", "value": value, "unit": "frames/s",
                "n_gpus": ws, "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3 / args.steps,
                "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "impl": "reference", "config": {"workload": cfg["desc"], "config_id": args.config},
                "cpu_baseline": {"value": value, "unit": "frames/s", "cores": 1, "kind": "oracle",
                                 "sample": "1 frame per step (resize + nine layers in fp64 + count)"},
                "e2e": {"value": value, "unit": "frames/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    S = min(cfg["streams"], 8)
    refs, params = {}, {}
    for s in range(S):
        r = synth.frames(video, [s] * 32, list(range(32)), ref=True)
        refs[s] = orc.reference(r, W, 100, 100)
        params[s] = synth.snm_weights(cfg["seed"], s)
    # frames: a mix that contains targets at the config's rate (planted schedule)
    n_distinct = 30
    frames = [(s, t) for t in range(n_distinct) for s in range(S)]
    cache = {}

    def step(i):
        s, t = frames[i % len(frames)]
        if (s, t) not in cache:
            cache[(s, t)] = synth.frame(video, s, t)
        f = cache[(s, t)]
        orc.filter_frames([f], W, [refs[s]], [DELTA], [params[s]], [C_LOW], [C_HIGH], [FD])

    for i in range(len(frames)):  # materialise the frames outside the timed region
        s, t = frames[i]
        cache[(s, t)] = synth.frame(video, s, t)
    for i in range(args.warmup):
        step(i)
    t0 = time.perf_counter()
    for i in range(args.steps):
        step(args.warmup + i)
    dt = time.perf_counter() - t0
    value = args.steps / dt
    return {"metric": METRIC, "value": value, "unit": "frames/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": dt * 1e3 / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u8 (SDD) / fp64 (SNM)", "data": "synthetic",
            "impl": "reference",
            "config": {"workload": cfg["desc"], "config_id": args.config},
            "cpu_baseline": {"value": value, "unit": "frames/s", "cores": 1, "kind": "oracle",
                             "sample": f"1 frame per step, round-robin over {S} streams x {n_distinct} frames of "
                                       f"the workload (targets at the config's rate)"},
            "e2e": {"value": value, "unit": "frames/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}


def spawn_ranks(args) -> int:
    """`python bench.py --gpus N` outside torchrun: build once here, then launch N ranks (one process per GPU) the
    way the driver does, with the build step disabled in the children, and relay rank 0's output."""
    import __graft_entry__ as ge
    ge.build()
    import socket
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    env = dict(os.environ, FFSVA_BENCH_PREBUILT="1")
    return subprocess.call(cmd, env=env)


def init_ranks(args, ws: int, rank: int, local: int):
    """Process group + build order under torchrun: every rank joins the group first, rank 0 builds (unless the
    launcher already did) while the others wait at a barrier, so no rank can load a half-written library."""
    if ws > 1:
        import torch
        import torch.distributed as dist
        if args.dist_backend == "nccl":
            if torch.cuda.device_count() < ws:
                raise SystemExit(f"--gpus {ws} with NCCL needs {ws} GPUs, found {torch.cuda.device_count()} "
                                 f"(--dist-backend gloo shares GPUs between ranks, for testing the N > 1 path)")
            torch.cuda.set_device(local)
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group("gloo")
    if os.environ.get("FFSVA_BENCH_PREBUILT") != "1" and rank == 0:
        import __graft_entry__ as ge
        ge.build()
    _barrier()


def main():
    ap = argparse.ArgumentParser(description=__doc__, formatter_class=argparse.RawDescriptionHelpFormatter)
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=2000)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--config", default="m2", choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend for N > 1 (gloo: ranks may share a GPU; a test mode)")
    ap.add_argument("--streams", type=int, default=3,
                    help="CUDA streams the timed steps alternate over (consecutive batches overlap)")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--cpu-frames", type=int, default=2400)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--online", default="30,auto",
                    help="comma-separated stream counts for the paced online validation (config m2); 'auto' = "
                         "a ladder of 55/70/85/90/95/100%% of the measured frames/s / 30, climbed until a count is not "
                         "sustained; empty to skip")
    ap.add_argument("--online-seconds", type=float, default=4.0, help="seconds per ladder rung")
    ap.add_argument("--online-tick-ms", type=float, default=0.0,
                    help="scheduler cycle period of the paced runs (0: 10 ms below 10 K streams, 25 ms below 30 K, "
                         "else 50 ms)")
    ap.add_argument("--online-confirm-seconds", type=float, default=30.0,
                    help="paced run that confirms a ladder's best rung (SURVEY.md §8(d): 30 s)")
    ap.add_argument("--online-tor", default="1,10,50",
                    help="target-occurrence sweep of the online ladder (config M4's TOR 1/10/50 %%); empty to skip")
    ap.add_argument("--online-tor-confirm-seconds", type=float, default=10.0)
    ap.add_argument("--online-tyolo", default="auto",
                    help="stream counts for a paced run of the full cascade with the T-YOLO stage (f1); 'auto' = "
                         "a ladder of 10/20/30/40/50%% of the measured frames/s / 30; empty to skip")
    args = ap.parse_args()
    if args.warmup < 3:
        ap.error("--warmup must be >= 3")
    ws, rank, local = dist_env()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(spawn_ranks(args))
    if ws != args.gpus and "WORLD_SIZE" in os.environ:
        ap.error(f"--gpus {args.gpus} but WORLD_SIZE={ws}")
    cfg = CONFIGS[args.config]
    if args.impl == "reference":  # the CPU oracle: rank 0 alone runs and prints it; the other ranks exit 0
        out = run_reference(args, cfg, ws, rank)
        if out is not None:
            print(json.dumps(out))
        return
    init_ranks(args, ws, rank, local)
    if args.dist_backend == "gloo":
        import torch
        local = local % max(1, torch.cuda.device_count())
    out = run_tyolo(args, cfg, ws, rank, local) if args.config == "tyolo" else run_ours(args, cfg, ws, rank, local)
    if rank == 0 and out is not None:
        print(json.dumps(out))
    if ws > 1:
        import torch.distributed as dist
        _barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
