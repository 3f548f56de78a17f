"""Per-layer device time of the T-YOLO stage (CUDA events, ffsva_tyolo_profile) on a batch of 720p frames, with
each layer's algorithmic FLOPs (2 x MACs of the convolution at its full resolution) and tensor-roofline fraction.

  python tools/tyolo_profile.py [--frames 256] [--iters 10]"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icpp_zhangcjzly18_b200 as ff  # noqa: E402
from synth import synth  # noqa: E402

# (H of the conv, Cin, Cout, k) of tiny-yolo-voc at 416x416
CONV = [(416, 3, 16, 3), (208, 16, 32, 3), (104, 32, 64, 3), (52, 64, 128, 3), (26, 128, 256, 3), (13, 256, 512, 3),
        (13, 512, 1024, 3), (13, 1024, 1024, 3), (13, 1024, 125, 1)]
FLOPS = [2 * h * h * ci * co * k * k for h, ci, co, k in CONV]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--frames", type=int, default=256)
    ap.add_argument("--iters", type=int, default=10)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "tyolo_profile.json"))
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    ctx = ff.Context(dev)
    W, H, n = 1280, 720, args.frames
    v = synth.Video(seed=3, width=W, height=H, period=4, on_len=2)
    frames = torch.empty((n, H, 3 * W), dtype=torch.uint8, device=dev)
    synth.frames_cuda(v, torch.zeros(n, dtype=torch.int32, device=dev), torch.arange(n, dtype=torch.int64, device=dev),
                      frames, H * 3 * W, 3 * W)
    st = ctx.open_stream(width=W, height=H)
    ty = ff.Tyolo(ctx, synth.tyolo_weights(1))
    items = [(st, frames[i], i) for i in range(n)]
    ty.profile(items, 2)
    ms = ty.profile(items, args.iters)
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["bf16_tflops"] if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else 1590.0
    rows = []
    for i, t in enumerate(ms):
        name = "resize" if i == 0 else f"L{i}"
        fl = FLOPS[i - 1] * n if i else 0
        tf = fl / (t / 1e3) / 1e12 if t > 0 else 0.0
        rows.append({"stage": name, "ms": t, "tflops": tf, "frac_of_peak": tf / peak})
        print(f"{name:7s} {t:8.3f} ms  {tf:8.1f} TFLOP/s  {tf / peak:.3f}")
    total = sum(ms)
    tot_fl = sum(FLOPS) * n
    res = {"frames": n, "ms_total": total, "frames_per_s": n / (total / 1e3), "gflop_per_frame": sum(FLOPS) / 1e9,
           "tflops": tot_fl / (total / 1e3) / 1e12, "peak_tflops": peak, "layers": rows}
    print(json.dumps({k: v for k, v in res.items() if k != "layers"}))
    with open(args.out, "w") as f:
        json.dump(res, f, indent=1)
    ty.destroy()
    ctx.close()


if __name__ == "__main__":
    main()
