"""Print the headline metrics of an ncu report (first kernel): time, DRAM, issue, warps, instructions, stalls."""
import csv
import subprocess
import sys

rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h, units = rows[0], rows[1]
for v in rows[2:]:
    print("==", v[h.index("Kernel Name")][:90])
    keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
            "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
            "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
            "smsp__issue_active.avg.pct_of_peak_sustained_active", "launch__occupancy_limit_registers",
            "launch__occupancy_limit_shared_mem", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
            "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"]
    for k in keys:
        if k in h:
            print(f"  {k} {v[h.index(k)]} {units[h.index(k)]}")
    st = [(float(v[i]), h[i]) for i in range(len(h)) if "warp_issue_stalled" in h[i] and h[i].endswith("per_warp_active.pct")
          and v[i] not in ("", "n/a")]
    for x, k in sorted(st, reverse=True)[:8]:
        print(f"  stall {k.split('stalled_')[1].split('_per')[0]} {x:.1f}%")

# warp-state sampling breakdown (share of all samples)
for v in rows[2:]:
    st = []
    for i, w in enumerate(h):
        if "pcsamp_warps_issue_stalled" in w and not w.endswith("not_issued"):
            try:
                st.append((float(v[i]), w.split("stalled_")[1]))
            except ValueError:
                pass
    tot = sum(x for x, _ in st) or 1.0
    print("  stalls:", ", ".join(f"{w} {x / tot * 100:.1f}%" for x, w in sorted(st, reverse=True)[:8]))
