"""Summarise ncu output into profiles/: the launch list (per-kernel share of the step) and
the `--set full` capture of the top kernels (DRAM/L2 traffic, throughput, stall reasons).

  python tools/ncu_summary.py --launches gpurun_out/launches_r1.csv --rep gpurun_out/prof_r1.ncu-rep \
      --queries-per-launch 16777216 --workload c2_T2^23_F64_Q2^26_uniform --out profiles/r1
"""
import argparse
import collections
import csv
import io
import json
import os
import re
import subprocess

METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum", "lts__t_sector_hit_rate.pct",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__t_sector_hit_rate.pct",
    "l1tex__throughput.avg.pct_of_peak_sustained_active", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "smsp__inst_executed.sum", "smsp__thread_inst_executed_per_inst_executed.ratio",
    "smsp__sass_average_branch_targets_threads_uniform.pct",
    "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "l1tex__data_pipe_lsu_wavefronts.sum.pct_of_peak_sustained_elapsed",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
    "lts__t_sectors.sum", "lts__t_sectors_srcunit_tex.sum", "lts__t_sectors_srcunit_ltcfabric.sum",
    "l1tex__data_pipe_lsu_wavefronts.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
]


def short(name):
    n = name.replace("(anonymous namespace)::", "").replace("::<unnamed>::", "::")
    n = re.sub(r"^(void )?<unnamed>::", "", n).replace("unnamed>::", "")
    n = n.replace("void ", "").replace("hm::", "").split("(")[0]
    return n.strip()


def launches(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.OrderedDict()
    for r in rows[hi + 1:]:
        v = float(r[vi].replace(",", ""))
        v *= {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "second": 1e6, "s": 1e6}.get(r[ui], 1.0)
        a = agg.setdefault(short(r[ki]), [0, 0.0])
        a[0] += 1
        a[1] += v
    tot = sum(a[1] for a in agg.values())
    return {k: {"launches": n, "total_us": us, "avg_us": us / n, "share": us / tot} for k, (n, us) in agg.items()}


def full(rep):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    h, units = rows[0], rows[1]
    out = []
    for r in rows[2:]:
        d = {"kernel": short(r[h.index("Kernel Name")])}
        for m in METRICS:
            if m in h:
                i = h.index(m)
                try:
                    d[m] = float(r[i].replace(",", ""))
                except ValueError:
                    d[m] = r[i]
                d[m + ".unit"] = units[i]
        stalls = {}
        for k in h:
            if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued"):
                try:
                    v = int(r[h.index(k)])
                except ValueError:
                    continue
                if v:
                    stalls[k.replace("smsp__pcsamp_warps_issue_stalled_", "")] = v
        tot = sum(stalls.values()) or 1
        d["stall_share"] = {k: round(v / tot, 3) for k, v in sorted(stalls.items(), key=lambda kv: -kv[1])[:8]}
        out.append(d)
    return out


def to_bytes(v, unit):
    return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--launches")
    ap.add_argument("--rep")
    ap.add_argument("--queries-per-launch", type=int, default=0)
    ap.add_argument("--workload", default="")
    ap.add_argument("--out", required=True)
    a = ap.parse_args()
    res = {"workload": a.workload}
    if a.launches:
        res["launch_list"] = launches(a.launches)
    if a.rep:
        res["full_capture"] = full(a.rep)
    json.dump(res, open(a.out + ".json", "w"), indent=1)
    # per-launch figures for bench.py's roofline (profiles/ncu_r2.json): traffic, L2 bytes,
    # sectors per request (memory divergence), warp coherence (P:L654 fn 4)
    tr_path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "ncu_r2.json")
    tr = json.load(open(tr_path)) if os.path.exists(tr_path) else {}
    for d in res.get("full_capture", []):
        k = d["kernel"].split("<")[0]
        rd = to_bytes(d.get("dram__bytes_read.sum", 0), d.get("dram__bytes_read.sum.unit", "byte"))
        wr = to_bytes(d.get("dram__bytes_write.sum", 0), d.get("dram__bytes_write.sum.unit", "byte"))
        # L2 traffic of the kernel = sectors its SMs (L1/TEX units) moved through L2 x 32 B
        # (lts__t_bytes is not in this ncu's full set; cross-die fabric sectors excluded)
        lts = float(d.get("lts__t_sectors_srcunit_tex.sum", 0) or 0) * 32.0
        ent = {"dram_bytes": rd + wr, "lts_bytes": lts,
               "source": os.path.basename(a.out) + ".json (ncu --set full --clock-control none, cold L2)"}
        if a.queries_per_launch:
            ent["dram_bytes_per_query"] = (rd + wr) / a.queries_per_launch
            ent["lts_bytes_per_query"] = lts / a.queries_per_launch
        sec = d.get("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum")
        req = d.get("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum")
        if isinstance(sec, float) and isinstance(req, float) and req:
            ent["sectors_per_request"] = sec / req
        r = d.get("smsp__thread_inst_executed_per_inst_executed.ratio")
        if isinstance(r, float):
            ent["warp_coherence"] = r / 32.0
        for key, m in (("branch_uniform_pct", "smsp__sass_average_branch_targets_threads_uniform.pct"),
                       ("l1_hit_pct", "l1tex__t_sector_hit_rate.pct"), ("lts_hit_pct", "lts__t_sector_hit_rate.pct"),
                       ("issue_active_pct", "smsp__issue_active.avg.pct_of_peak_sustained_active"),
                       ("l1_wavefront_pct", "l1tex__data_pipe_lsu_wavefronts.sum.pct_of_peak_sustained_elapsed"),
                       ("lts_pct", "lts__throughput.avg.pct_of_peak_sustained_elapsed"),
                       ("dram_pct", "dram__throughput.avg.pct_of_peak_sustained_elapsed")):
            v = d.get(m)
            if isinstance(v, float):
                ent[key] = v
        tv, tu = d.get("gpu__time_duration.sum"), d.get("gpu__time_duration.sum.unit", "nsecond")
        if isinstance(tv, float):
            ent["ncu_time_s"] = tv * {"ns": 1e-9, "nsecond": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3,
                                      "msecond": 1e-3, "s": 1.0, "second": 1.0}.get(tu, 1e-9)
        # L1 data-pipe (LSU) wavefronts per launch: global/local loads and stores, shared-memory
        # accesses, atomics and shuffles all pass this pipe (1 wavefront per cycle per SM)
        for key, m in (("lsu_wavefronts", "l1tex__data_pipe_lsu_wavefronts.sum"),
                       ("lsu_wavefronts_shared", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum")):
            v = d.get(m)
            if isinstance(v, float):
                ent[key] = v
        st = d.get("stall_share")
        if isinstance(st, dict) and "long_scoreboard" in st:
            ent["long_scoreboard_stall_share"] = st["long_scoreboard"]
        tr.setdefault(a.workload, {})[k] = ent  # the newest capture supersedes
    json.dump(tr, open(tr_path, "w"), indent=1)
    with open(a.out + ".md", "w") as f:
        f.write(f"# ncu summary {os.path.basename(a.out)} — {a.workload}\n\n")
        if "launch_list" in res:
            f.write("## Launch list (`--metrics gpu__time_duration.sum --clock-control none`; cold, serialised: compare shares)\n\n")
            f.write("| kernel | launches | avg µs | share |\n|---|---|---|---|\n")
            for k, v in sorted(res["launch_list"].items(), key=lambda kv: -kv[1]["share"]):
                f.write(f"| {k} | {v['launches']} | {v['avg_us']:.1f} | {v['share']:.3f} |\n")
        if "full_capture" in res:
            f.write("\n## `--set full` captures\n\n")
            for d in res["full_capture"]:
                f.write(f"### {d['kernel']}\n\n")
                for m in METRICS:
                    if m in d:
                        f.write(f"- {m}: {d[m]} {d.get(m + '.unit', '')}\n")
                f.write(f"- stall share (pc sampling): {d['stall_share']}\n\n")
    print(open(a.out + ".md").read())
