"""Summarise ncu outputs for profiles/: per-kernel key metrics of a --set full capture, and per-class
time shares of a gpu__time_duration launch list.

  python tools/ncu_summary.py full gpurun_out/r01_prof.ncu-rep > profiles/r01_ncu_full_summary.csv
  python tools/ncu_summary.py launches gpurun_out/r01_launches.csv > profiles/r01_launch_shares.csv
"""
import collections
import csv
import io
import subprocess
import sys

FULL = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active", "lts__t_bytes.sum",
        "launch__registers_per_thread", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "smsp__pcsamp_warps_issue_stalled_barrier",
        "smsp__pcsamp_warps_issue_stalled_wait", "smsp__pcsamp_warps_issue_stalled_long_scoreboard",
        "smsp__pcsamp_warps_issue_stalled_math_pipe_throttle"]


def full(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    idx = [(h, hdr.index(h)) for h in FULL if h in hdr]
    w = csv.writer(sys.stdout)
    w.writerow([f"{h} [{units[i]}]" if units[i] else h for h, i in idx])
    for r in rows[2:]:
        w.writerow([r[i] for _, i in idx])


def launches(path):
    lines = [l for l in open(path) if not l.startswith("==")]
    rows = list(csv.DictReader(io.StringIO("".join(lines))))
    t = collections.defaultdict(float)
    n = collections.Counter()
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        k = r["Kernel Name"].split("(")[0].replace("void ", "")
        t[k] += float(r["Metric Value"])
        n[k] += 1
    tot = sum(t.values())
    w = csv.writer(sys.stdout)
    w.writerow(["kernel", "launches", "total_ns", "avg_ns", "share"])
    for k, v in sorted(t.items(), key=lambda kv: -kv[1]):
        w.writerow([k, n[k], f"{v:.0f}", f"{v / n[k]:.0f}", f"{v / tot:.4f}"])


if __name__ == "__main__":
    {"full": full, "launches": launches}[sys.argv[1]](sys.argv[2])
