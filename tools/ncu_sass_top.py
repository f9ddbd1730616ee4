"""Top SASS instructions of one kernel in an ncu --set full report (stall samples, executed
instructions, L1/L2 traffic per instruction).   python tools/ncu_sass_top.py REP [N] [KERNEL_REGEX]"""
import csv
import io
import re
import subprocess
import sys

rep, n = sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 40
cmd = ["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"]
if len(sys.argv) > 3:
    cmd += ["-k", "regex:" + sys.argv[3]]
txt = subprocess.run(cmd, capture_output=True, text=True).stdout
lines = txt.splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith('"Address"'))
rows = list(csv.reader(io.StringIO("\n".join(lines[start:]))))
h = rows[0]
c = {k: i for i, k in enumerate(h)}


def f(r, k):
    try:
        return float(r[c[k]].replace(",", "")) if k in c and r[c[k]] not in ("", "-") else 0.0
    except ValueError:
        return 0.0


body = [r for r in rows[1:] if len(r) == len(h)]
tot = sum(f(r, "Warp Stall Sampling (All Samples)") for r in body) or 1
tot_wf = sum(f(r, "L1 Wavefronts Shared") for r in body)
tot_l2 = sum(f(r, "L2 Theoretical Sectors Global") for r in body)
tot_tag = sum(f(r, "L1 Tag Requests Global") for r in body)
print(f"samples {tot:.0f}  smem wavefronts {tot_wf:.3g}  L1 tag req global {tot_tag:.3g}  L2 sectors {tot_l2:.3g}")
for i, r in enumerate(body):
    r.append(i)
body.sort(key=lambda r: -f(r, "Warp Stall Sampling (All Samples)"))
for r in body[:n]:
    stalls = {k[6:]: f(r, k) for k in h if k.startswith("stall_") and "Not Issued" not in k}
    top = sorted(stalls.items(), key=lambda kv: -kv[1])[:2]
    print(f"{r[-1]:5d} {f(r,'Warp Stall Sampling (All Samples)')/tot*100:5.1f}% ex={f(r,'Instructions Executed'):.3g} "
          f"tag={f(r,'L1 Tag Requests Global'):.3g} l2s={f(r,'L2 Theoretical Sectors Global'):.3g} "
          f"swf={f(r,'L1 Wavefronts Shared'):.3g} {r[c['Source']].strip()[:60]:60s} {top}")
