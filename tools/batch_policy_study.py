"""f4: the paper's batch-mechanism comparison (§5.4, Figs. 9-10) on B200: static batch,
feedback queue and dynamic batching, BatchSize sweep, 10 synthetic 720p streams at TOR 0.203 and 0.980, each
run saturated through the online runtime (paper_conf_icpp_zhangcjzly18_b200.online.run_unpaced).

  python tools/batch_policy_study.py [--seconds 2] [--out gpurun_out/batch_policy]

Writes <out>.json (every run) and <out>.md (throughput and mean latency tables)."""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icpp_zhangcjzly18_b200 as ff  # noqa: E402
from paper_conf_icpp_zhangcjzly18_b200.online import run_unpaced  # noqa: E402
from synth import synth  # noqa: E402

POLICIES = ["static", "feedback", "dynamic"]
TORS = {"0.203": 61, "0.980": 294}  # target frames per 300-frame period (Fig. 9: 0.203, Fig. 10: 0.980)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--seconds", type=float, default=2.0)
    ap.add_argument("--streams", type=int, default=10)
    ap.add_argument("--batch", default="1,2,5,10,20,30,50")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "batch_policy"))
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    ctx = ff.Context(dev)
    W, H, P, NF = 1280, 720, 3 * 1280, 300
    batches = [int(b) for b in args.batch.split(",")]
    runs = []
    for tor, on_len in TORS.items():
        video = synth.Video(seed=1404, width=W, height=H, period=300, on_len=on_len)
        content = []
        for s in range(args.streams):
            pool = torch.empty((NF, H, P), dtype=torch.uint8, device=dev)
            synth.frames_cuda(video, torch.full((NF,), s, dtype=torch.int32, device=dev),
                              torch.arange(NF, dtype=torch.int64, device=dev), pool, H * P, P)
            content.append(pool)
        refs = []
        for s in range(args.streams):
            r = torch.empty((32, H, P), dtype=torch.uint8, device=dev)
            synth.frames_cuda(video, torch.full((32,), s, dtype=torch.int32, device=dev),
                              torch.arange(32, dtype=torch.int64, device=dev), r, H * P, P, ref=True)
            refs.append(r)
        for bs in batches:
            streams = []
            for s in range(args.streams):
                st = ctx.open_stream(width=W, height=H, snm_batch=bs)
                st.set_reference(refs[s])
                st.snm_load(synth.snm_weights(1404, s))
                streams.append(st)
            for pol in POLICIES:
                r = run_unpaced(ctx, streams, content, NF, args.seconds, policy=pol)
                r.update(tor=float(tor), batch_size=bs)
                runs.append(r)
                print(json.dumps(r), flush=True)
            for st in streams:
                st.close()
        del content, refs
        torch.cuda.empty_cache()
    ctx.close()
    with open(args.out + ".json", "w") as f:
        json.dump(runs, f, indent=1)
    lines = ["# f4 batch-mechanism study (PAPER.md §5.4): %d streams 1280x720, saturated online runtime, %.1f s "
             "per run, B200" % (args.streams, args.seconds), ""]
    for tor in TORS:
        for key, name in [("fps", "throughput (decided frames/s)"), ("latency_mean_ms", "mean latency (ms)"),
                          ("mean_snm_batch", "mean SNM batch (frames)")]:
            lines += [f"## TOR {tor}: {name}", "", "| BatchSize | " + " | ".join(POLICIES) + " |",
                      "|---|" + "---|" * len(POLICIES)]
            for bs in batches:
                row = [next(r[key] for r in runs if r["tor"] == float(tor) and r["batch_size"] == bs
                            and r["policy"] == p) for p in POLICIES]
                lines.append(f"| {bs} | " + " | ".join(f"{v:,.1f}" for v in row) + " |")
            lines.append("")
    with open(args.out + ".md", "w") as f:
        f.write("\n".join(lines))
    print("\n".join(lines))


if __name__ == "__main__":
    main()
