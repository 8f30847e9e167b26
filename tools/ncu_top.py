"""Print the top stall sites and headline metrics of one kernel in an ncu report (reading aid).
  python tools/ncu_top.py REPORT [n]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
ntop = int(sys.argv[2]) if len(sys.argv) > 2 else 20
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(src)))
h = r[1]
rows = r[2:]
i_s = h.index("Warp Stall Sampling (All Samples)")
tot = sum(float(x[i_s] or 0) for x in rows) or 1
for x in sorted(rows, key=lambda x: -float(x[i_s] or 0))[:ntop]:
    print(x[0][-5:], x[1][:72], x[i_s], round(float(x[i_s]) / tot, 3))
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
h, u, v = r[0], r[1], r[2]
for k in ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
          "dram__throughput.avg.pct_of_peak_sustained_elapsed",
          "sm__ops_path_tensor_op_utcimma_src_int8_sparsity_off.avg.pct_of_peak_sustained_elapsed",
          "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", "lts__t_bytes.sum",
          "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread"]:
    if k in h:
        print(k, u[h.index(k)], v[h.index(k)])
for i, k in enumerate(h):
    if "pcsamp_warps_issue_stalled" in k and "not_issued" not in k and float(v[i] or 0) > 200:
        print(k, v[i])
