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
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "200", "-i", str(self.device)], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
            return
        self.th = threading.Thread(target=self._read, daemon=True)
        self.th.start()

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
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


# ---------------------------------------------------------------------------------------------- our arm

def run_ours(args, cfg, ws, rank, local):
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_zhangcjzly18_b200 as ff
    from paper_conf_icpp_zhangcjzly18_b200 import ffsva as ffb
    from synth import synth

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if ws > 1:
        dist.init_process_group("nccl", device_id=dev)
    W, H, P = cfg["W"], cfg["H"], 3 * cfg["W"]
    fbytes = H * P
    if cfg.get("shard"):
        lo, hi = rank * cfg["streams"] // ws, (rank + 1) * cfg["streams"] // ws
        sids = list(range(lo, hi))
    else:
        sids = [rank * cfg["streams"] + s for s in range(cfg["streams"])]
    S, PF, SF = len(sids), cfg["pool_frames"], cfg["step_frames"]
    video = synth.Video(seed=cfg["seed"], width=W, height=H, period=cfg["period"], on_len=cfg["on_len"])
    ctx = ff.Context(dev)
    streams = []
    for s in sids:
        st = ctx.open_stream(width=W, height=H, delta_diff=cfg.get("delta", DELTA), c_low=C_LOW, c_high=C_HIGH,
                             filter_degree=FD,
                             snm_batch=BATCH)
        refs = torch.empty((32, H, P), dtype=torch.uint8, device=dev)
        synth.frames_cuda(video, torch.full((32,), s, dtype=torch.int32, device=dev),
                          torch.arange(32, dtype=torch.int64, device=dev), refs, fbytes, P, ref=True)
        st.set_reference(refs)
        del refs
        st.snm_load(synth.snm_weights(cfg["seed"], s))
        streams.append(st)
    # frame pool: stream-major, pool[s][t]
    pool = torch.empty((S, PF, H, P), dtype=torch.uint8, device=dev)
    for k, s in enumerate(sids):
        synth.frames_cuda(video, torch.full((PF,), s, dtype=torch.int32, device=dev),
                          torch.arange(PF, dtype=torch.int64, device=dev), pool[k], fbytes, P)
    torch.cuda.synchronize()
    # prepared batches: batch j = frames [j*SF, (j+1)*SF) of every stream (one second of video)
    nbatches = max(1, PF // SF)
    batches = []
    for j in range(nbatches):
        items = [(streams[k], pool[k, j * SF + i], j * SF + i) for k in range(S) for i in range(SF)]
        batches.append(ctx.prepare(items))
    frames_per_step = S * SF
    planted = [sum(synth.planted(video, s, j * SF, (j + 1) * SF) for s in sids) for j in range(nbatches)]
    cs = torch.cuda.Stream(device=dev)
    stats_dev = torch.zeros((max(1, S), ffb.NSTAT), dtype=torch.int64, device=dev)
    gathered = torch.zeros((ws * max(1, S), ffb.NSTAT), dtype=torch.int64, device=dev) if ws > 1 else None

    # correctness gate before timing: SDD pass count == planted count on every batch (P8 at full size)
    for j, b in enumerate(batches):
        b.launch(cs)
        r = b.fetch(cs)
        expect = planted[j] if cfg.get("delta", DELTA) == DELTA else frames_per_step
        if int(r["sdd_pass"].sum()) != expect:
            raise RuntimeError(f"batch {j}: SDD passed {int(r['sdd_pass'].sum())} != expected {expect}")
        planted[j] = expect
    ctx.stats(reset=True)

    # consecutive steps alternate over --streams CUDA streams (different prepared batches, own buffers): step i+1's
    # K1 starts while step i's K1 tail, K3 and K4 still run (the per-stream statistics are order-independent atomics)
    nstr = max(1, min(args.streams, nbatches))
    css = [cs] + [torch.cuda.Stream(device=dev) for _ in range(nstr - 1)]

    def step(i):
        batches[i % nbatches].launch(css[i % nstr])

    for i in range(args.warmup):
        step(i)
    torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)
    launches0 = ff.ffsva_kernel_launches()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    with torch.cuda.stream(cs):
        e0.record(cs)
        for s2 in css[1:]:
            s2.wait_event(e0)
        for i in range(args.steps):
            step(args.warmup + i)
        for s2 in css[1:]:  # the timed region ends when every stream's last step is done
            ev = torch.cuda.Event()
            ev.record(s2)
            cs.wait_event(ev)
        # a8 reporting: per-stream statistics to a device tensor, all-gathered over NCCL when sharded
        ffb.ffsva_stats_copy(local, stats_dev.data_ptr(), S, False, False, cs.cuda_stream)
        if ws > 1:
            dist.all_gather_into_tensor(gathered, stats_dev)
        e1.record(cs)
    torch.cuda.synchronize()
    launches = ff.ffsva_kernel_launches() - launches0
    if ws > 1:
        dist.barrier()
    clk = clocks.stop()
    ms = e0.elapsed_time(e1)
    t = torch.tensor([ms], dtype=torch.float64, device=dev)
    if ws > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max = float(t.item())
    total_frames = frames_per_step * args.steps * ws
    value = total_frames / (ms_max / 1e3)
    st_rows = stats_dev.cpu().numpy()
    if int(st_rows[:, 0].sum()) != frames_per_step * (args.warmup + args.steps):
        raise RuntimeError("per-stream frame counters disagree with the frames launched")

    # ---- per-kernel device times (CUDA events on the launching stream) for the roofline
    k_ms = ffb.ffsva_batch_profile([b.handle for b in batches], max(2, min(10, 30 // nbatches + 1)), cs.cuda_stream)
    r_last = batches[0].fetch(cs)
    m_avg = float(np.mean(planted))
    k1_bytes = frames_per_step * (3 * W * H + 9) + m_avg * 7500
    hbm_peak, tf_peak, peak_kind = measured_peaks()
    achieved = k1_bytes / (k_ms[0] / 1e3) / 1e9
    traffic = ncu_traffic(args.config)

    # ---- end to end through the public API with HOST buffers (pinned), H2D + D2H inside the timed region
    e2e = None
    if not args.no_e2e:
        n_e2e = max(1, min(args.steps, args.e2e_steps))
        pinned = torch.empty((S, SF, H, P), dtype=torch.uint8).pin_memory()
        pinned.copy_(pool[:, :SF].cpu())
        items = [(streams[k], pinned[k, i].data_ptr(), i) for k in range(S) for i in range(SF)]
        ctx.filter_batch(items, stream=cs, host=True)  # warm-up (ring allocation)
        torch.cuda.synchronize()
        if ws > 1:
            dist.barrier()
        h0, h1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        h0.record(cs)
        for _ in range(n_e2e):
            res = ctx.filter_batch(items, stream=cs, host=True)
        h1.record(cs)
        torch.cuda.synchronize()
        te = torch.tensor([h0.elapsed_time(h1)], dtype=torch.float64, device=dev)
        if ws > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        e2e_val = frames_per_step * n_e2e * ws / (float(te.item()) / 1e3)
        e2e = {"value": e2e_val, "unit": "frames/s", "h2d_bytes_per_step": int(frames_per_step * fbytes),
               "d2h_bytes_per_step": int(frames_per_step * ffb.RESULT_DTYPE.itemsize), "steps": n_e2e,
               "path": "ffsva_filter_batch_host (pinned host frames -> 2-chunk device ring, copies overlapped "
                       "with K1)"}
        del pinned

    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(cfg, video, sids, pool, args.cpu_frames)

    # ---- online validation of "sustained 30-FPS streams" (paced arrivals through the online runtime)
    online = None
    if args.online and args.config == "m2":
        online = online_validation(args, ctx, video, sids, pool, value / ws, dev, cs, ws)

    out = None
    if rank == 0:
        out = {
            "metric": METRIC, "value": value, "unit": "frames/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u8 (SDD) / bf16-fp32 (SNM)", "data": "synthetic",
            "config": {"workload": cfg["desc"], "config_id": args.config, "streams_per_gpu": S,
                       "frames_per_step": frames_per_step * ws, "frame_bytes": fbytes,
                       "pool_bytes_per_gpu": int(S * PF * fbytes),
                       "l2": "inputs larger than L2: each step reads a different %.2f GB slice of the pool"
                             % (frames_per_step * fbytes / 1e9),
                       "parallelism": f"stream-sharded x{ws} (weak: {S} streams per GPU)",
                       "batch_size": BATCH, "delta_diff": DELTA, "c_low": C_LOW, "c_high": C_HIGH,
                       "filter_degree": FD, "seed": cfg["seed"], "cuda_streams": nstr},
            "sustained_streams_30fps": int(value // 30),
            "sdd_pass_per_step": m_avg,
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
            "online": online,
        }
        if args.config == "snm":  # K4 is this workload's dominant kernel: its tensor roofline is the line's
            out["sdd_roofline"] = out["roofline"]
            out["roofline"] = dict(out["snm_roofline"], kernel_ms=out["sdd_roofline"]["kernel_ms"],
                                   k4_share_of_step=k_ms[2] / max(1e-9, sum(k_ms)))
    for b in batches:
        b.destroy()
    ctx.close()
    if ws > 1:
        dist.destroy_process_group()
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

    N > 1: every rank runs the same per-GPU counts on its own GPU at the same time (streams are sharded, no frame
    crosses GPUs); a count is sustained only if it is sustained on every rank (all-reduce MIN of the verdicts, so
    the ranks also climb their ladders in lock step), and the whole-job count is N x the per-GPU count."""
    import torch
    import torch.distributed as dist

    from paper_conf_icpp_zhangcjzly18_b200.online import run_paced
    from synth import synth
    W, H, P = video.width, video.height, 3 * video.width
    counts, ladder = [], []
    for tok in args.online.split(","):
        tok = tok.strip()
        if tok == "auto":  # a ladder of fractions of the offline capacity, climbed until a count is not sustained
            ladder = [max(31, int(f * value / 30)) for f in (0.55, 0.7, 0.85, 0.9, 0.95)]
        elif tok:
            counts.append(int(tok))
    nc = len(sids)
    refs = []
    for k, s in enumerate(sids):
        r = torch.empty((32, H, P), dtype=torch.uint8, device=dev)
        synth.frames_cuda(video, torch.full((32,), s, dtype=torch.int32, device=dev),
                          torch.arange(32, dtype=torch.int64, device=dev), r, H * P, P, ref=True)
        refs.append(r)
    # full three-filter cascade (f1: SDD -> SNM -> T-YOLO, random-init T-YOLO weights) at these stream counts
    ty_counts = []
    ty_ladder = []
    for tok in args.online_tyolo.split(","):
        tok = tok.strip()
        if tok == "auto":  # T-YOLO (~55 K frames/s) sees the SNM survivors, a few % of the frames at TOR 10 %:
            ty_ladder = [max(31, int(f * value / 30)) for f in (0.1, 0.2, 0.3, 0.4, 0.5)]  # climbed like SDD+SNM's
        elif tok:
            ty_counts.append(int(tok))
    results = []
    opened = []
    runs = ([(S, False) for S in counts] + [(S, False) for S in ladder] + [(S, True) for S in ty_counts] +
            [(S, True) for S in ty_ladder])
    ty = None
    if ty_counts or ty_ladder:
        import paper_conf_icpp_zhangcjzly18_b200 as ff
        ty = ff.Tyolo(ctx, synth.tyolo_weights(video.seed))
    ty_warm = False
    ladder_failed = ty_ladder_failed = False
    for S, with_ty in runs:
        if (S in ladder and not with_ty and ladder_failed) or (S in ty_ladder and with_ty and ty_ladder_failed):
            continue  # a ladder stops at its first count that is not sustained
        t_setup = time.perf_counter()
        while len(opened) < S:
            i = len(opened)
            st = ctx.open_stream(width=W, height=H, delta_diff=DELTA, c_low=C_LOW, c_high=C_HIGH, filter_degree=FD,
                                 snm_batch=BATCH, q_sdd=2, q_snm=10)
            st.set_reference(refs[i % nc])
            st.snm_load(synth.snm_weights(video.seed, 100000 + i))
            opened.append(st)
        setup_s = time.perf_counter() - t_setup
        if with_ty and not ty_warm:  # outside the paced window: the first T-YOLO launches load their modules
            ty.run([(opened[0], pool[0][t], t) for t in range(2)], target_class=14, thresh=0.2)
            ty_warm = True
        # cycles of 10 ms, 25 ms from 10 K streams on (the driver's per-cycle work over all cameras is amortised)
        res = run_paced(ctx, opened[:S], [pool[i % nc] for i in range(S)], pool.shape[1], args.online_seconds,
                        cuda_stream=cs, tyolo=ty if with_ty else None, tick_s=0.010 if S < 10000 else 0.025)
        res["stream_setup_s"] = setup_s
        if ws > 1:
            ok = torch.tensor([1 if res["sustained"] else 0], dtype=torch.int32, device=dev)
            dist.all_reduce(ok, op=dist.ReduceOp.MIN)
            res["sustained_this_rank"] = res["sustained"]
            res["sustained"] = bool(ok.item())
            res["streams_per_gpu"], res["streams"] = S, S * ws
        results.append(res)
        if S in ladder and not with_ty and not res["sustained"]:
            ladder_failed = True
        if S in ty_ladder and with_ty and not res["sustained"]:
            ty_ladder_failed = True
    closed = set(id(st) for st in opened)
    for st in opened:
        st.close()
    ctx.streams = [st for st in ctx.streams if id(st) not in closed]  # (list.remove per stream is O(S^2))
    if ty is not None:
        ty.destroy()
    best = max([r["streams"] for r in results if r["sustained"] and "stages" not in r], default=0)
    best_ty = max([r["streams"] for r in results if r["sustained"] and "stages" in r], default=0)
    return {"runs": results, "max_sustained_streams_validated": best,
            "max_sustained_streams_validated_with_tyolo": best_ty,
            "policy": "q_sdd 2, q_snm 10, q_tyolo 2, BatchSize 30, num_t-yolo 4 (PAPER.md L173, L217, L219); "
                      "latency budget p99 <= 1 s"}


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


def main():
    ap = argparse.ArgumentParser(description=__doc__, formatter_class=argparse.RawDescriptionHelpFormatter)
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=2000)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--config", default="m2", choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--streams", type=int, default=2,
                    help="CUDA streams the timed steps alternate over (consecutive batches overlap)")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--cpu-frames", type=int, default=2400)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--online", default="30,auto",
                    help="comma-separated stream counts for the paced online validation (config m2); 'auto' = "
                         "a ladder of 55/70/85/90/95%% of the measured frames/s / 30, climbed until a count is not "
                         "sustained; empty to skip")
    ap.add_argument("--online-seconds", type=float, default=4.0)
    ap.add_argument("--online-tyolo", default="2000,auto",
                    help="stream counts for a paced run of the full cascade with the T-YOLO stage (f1); 'auto' = "
                         "a ladder of 10/20/30/40/50%% of the measured frames/s / 30; empty to skip")
    args = ap.parse_args()
    if args.warmup < 3:
        ap.error("--warmup must be >= 3")
    ws, rank, local = dist_env()
    cfg = CONFIGS[args.config]
    if args.impl == "reference":
        out = run_reference(args, cfg, ws, rank)
    else:
        import __graft_entry__ as ge
        if rank == 0:
            ge.build()
        if ws > 1:
            # other ranks wait for rank 0's build (the .so must exist before they load it)
            while not os.path.exists(os.path.join(ROOT, "paper_conf_icpp_zhangcjzly18_b200", "lib", "libffsva.so")):
                time.sleep(0.5)
        out = run_tyolo(args, cfg, ws, rank, local) if args.config == "tyolo" else run_ours(args, cfg, ws, rank, local)
    if rank == 0 and out is not None:
        print(json.dumps(out))


if __name__ == "__main__":
    main()
