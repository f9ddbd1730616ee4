"""Print a compact per-kernel summary of an ncu --set full report: duration, throughputs,
occupancy and the top warp-stall reasons.   python tools/ncu_stalls.py REPORT.ncu-rep"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h = rows[0]
col = {n: i for i, n in enumerate(h)}
want = [
    ("gpu__time_duration.sum", "us", 1e-3),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "dram%", 1),
    ("lts__t_sectors.avg.pct_of_peak_sustained_elapsed", "l2%", 1),
    ("l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_active", "l1wf%", 1),
    ("sm__issue_active.avg.pct_of_peak_sustained_active", "issue%", 1),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "occ%", 1),
    ("dram__bytes_read.sum", "rdMB", 1e-6),
    ("dram__bytes_write.sum", "wrMB", 1e-6),
]
for r in rows[2:]:
    name = r[col["Kernel Name"]]
    name = name[name.find("k_"):][:40] if "k_" in name else name[:40]
    out = []
    for m, lab, sc in want:
        if m in col:
            try:
                v = float(r[col[m]].replace(",", ""))
                if m == "gpu__time_duration.sum" and "msecond" in rows[1][col[m]]:
                    sc = 1e3
                elif m == "gpu__time_duration.sum" and "usecond" in rows[1][col[m]]:
                    sc = 1
                out.append(f"{lab}={v * sc:.1f}")
            except ValueError:
                pass
    st = []
    for i, n in enumerate(h):
        if n.startswith("smsp__average_warps_issue_stalled_") and n.endswith("_per_issue_active.ratio"):
            try:
                st.append((float(r[i]), n[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
            except ValueError:
                pass
    st.sort(reverse=True)
    print(f"{name:40s} " + " ".join(out))
    print("    stalls/issue: " + ", ".join(f"{n}={v:.1f}" for v, n in st[:6]))
