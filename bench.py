#!/usr/bin/env python
"""Harmonia B200 benchmark — point queries/s of the batched search path (BASELINE config 2
by default: 2^23 uint64 keys, fanout 64, 2^26 uniform point queries per GPU).

One step = one harmonia_search_batch call over the whole batch: PSA (histogram, scan,
scatter) + NTG search + return to caller order, with queries and results resident in HBM.
`e2e` repeats the measurement through harmonia_search_batch_host with pinned host buffers
(H2D of the queries and D2H of the results inside the timed region).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C] [--impl harmonia|reference]
  torchrun --nproc-per-node N bench.py --gpus N     (replicated tree, batch split, no collective)

Prints ONE JSON line on rank 0 (see DESIGN.md §8 for every field).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import harmonia_gen as gen  # noqa: E402

CONFIGS = {
    1: dict(name="c1_T2^16_F16_Q2^20_uniform", T=1 << 16, F=16, Q=1 << 20, dist="uniform"),
    2: dict(name="c2_T2^23_F64_Q2^26_uniform", T=1 << 23, F=64, Q=1 << 26, dist="uniform"),
    3: dict(name="c3_T2^26_F64_Q2^26_zipf", T=1 << 26, F=64, Q=1 << 26, dist="zipf"),
    4: dict(name="c4_T2^28_F64_Q2^27_uniform_replicated", T=1 << 28, F=64, Q=1 << 27, dist="uniform"),
    # config 5: 2^32 keys range-partitioned over 8 shards of 2^29 (rank p holds shard p), queries
    # uniform over the running ranks' keys and routed, update batches of 2^22 ops (5 % insert,
    # 5 % delete, 90 % update) interleaved 1:1 with the query batches
    # The shard is bulk-loaded at fill 0.69, the occupancy of the paper's insertion-built trees
    # ("half full", P:L592 fn 3; C-A6), so update batches go in place when leaves have room.
    5: dict(name="c5_T2^32_8shards_F64_fill0.69_Q2^27_uniform_partitioned_updates", T=1 << 32, F=64, Q=1 << 27,
            dist="uniform", shards=8, ops=1 << 22, fill=0.69),
}
METRIC = "point queries/sec (G q/s) at 1/2/4/8 B200; % of L2/HBM roofline"
UNIT = "G q/s"
PAPER_TITANV_GQS = 3.6  # P:L40, L592 (Fig 11) — context only, other hardware


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--impl", default="harmonia", choices=["harmonia", "reference"])
    ap.add_argument("--fanout", type=int, default=0)
    ap.add_argument("--keys", type=int, default=0, help="override T (log2 if < 64)")
    ap.add_argument("--queries", type=int, default=0, help="override Q per GPU (log2 if < 64)")
    ap.add_argument("--dist", default="", help="uniform|zipf|sorted_run")
    ap.add_argument("--fill", type=float, default=1.0)
    ap.add_argument("--group-size", type=int, default=0)
    ap.add_argument("--psa-bits", type=int, default=0)
    ap.add_argument("--window", type=int, default=0)
    ap.add_argument("--smem-levels", type=int, default=0)
    ap.add_argument("--flags", type=int, default=0)
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--mode", default="replicated", choices=["replicated", "partitioned", "peer"])
    ap.add_argument("--sweep", default="", help="comma list of k=v option sets separated by ';' (diagnostics)")
    ap.add_argument("--no-extra", action="store_true", help="skip the c4 / c3-fanout extra lines (default run)")
    ap.add_argument("--slices", type=int, default=4, help="partitioned mode: exchange/search overlap slices")
    ap.add_argument("--extra-steps", type=int, default=10)
    return ap.parse_args()


def workload(a):
    c = dict(CONFIGS[a.config])
    if a.fanout:
        c["F"] = a.fanout
    if a.keys:
        c["T"] = 1 << a.keys if a.keys < 64 else a.keys
    if a.queries:
        c["Q"] = 1 << a.queries if a.queries < 64 else a.queries
    if a.dist:
        c["dist"] = a.dist
    if a.keys or a.queries or a.fanout or a.dist:
        c["name"] = f"custom_T{c['T']}_F{c['F']}_Q{c['Q']}_{c['dist']}"
    return c


def make_queries(keys, Q, dist, rank):
    if dist == "uniform":
        return gen.uniform_queries(keys, Q, start=rank * Q)
    if dist == "zipf":
        return gen.zipf_queries(keys, Q, start=rank * Q)
    if dist == "sorted_run":
        return gen.sorted_run_queries(keys, Q, seed=gen.SEED_QUERY + rank)
    raise ValueError(dist)


def host_threads():
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


# ------------------------------------------------------------------------------ clocks
class ClockSampler:
    """NVML sampling of SM clock and throttle reasons during the timed region."""

    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, dev_index, period=0.01):
        self.samples, self.reasons, self.ok = [], set(), False
        self.period = period
        try:
            import pynvml

            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(dev_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover
            self.err = str(e)
            self.max_mhz = None

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self._stop = threading.Event()
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *exc):
        if self.ok:
            self._stop.set()
            self._t.join()

    def summary(self):
        if not self.ok:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "error": getattr(self, "err", "")}
        med = float(np.median(self.samples)) if self.samples else None
        return {"sm_mhz": med, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons - {"gpu_idle"}),
                "samples": len(self.samples)}


# ------------------------------------------------------------------------------ CPU legs
def cpu_model() -> str:
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def _best_rate(fn, n, runs=5):
    """queries/s of fn(n): one warm-up, then the best of `runs`."""
    fn(n)
    best = 1e30
    for _ in range(runs):
        t0 = time.perf_counter()
        fn(n)
        best = min(best, time.perf_counter() - t0)
    return n / best, best


def _size_for(fn, seconds, cap):
    """A sample size whose run takes about `seconds` (calibrated on 2^16 queries)."""
    n0 = min(cap, 1 << 16)
    t0 = time.perf_counter()
    fn(n0)
    dt = max(time.perf_counter() - t0, 1e-6)
    return int(max(n0, min(cap, n0 * seconds / dt)))


def cpu_baselines(keys, vals, q, seconds, fanout):
    """The CPU oracle as it stands, on the host cores of this box: O1
    std::lower_bound + value fetch and the O2 pointer B+tree (the paper's regular B+tree,
    P:L120/L218; built by sorted-order insertion, fanout F), each with 1 thread and with
    every host thread, best of 5 after 1 warm-up on a bounded sample of the batch."""
    import oracle

    nth = host_threads()
    per = max(0.2, seconds / 24.0)  # 4 legs x 6 runs
    out = {"cores": nth, "cpu_model": cpu_model(), "method": "best of 5 after 1 warm-up"}
    f1 = lambda n: oracle.sorted_search(keys, vals, q[:n], 1)
    fN = lambda n: oracle.sorted_search(keys, vals, q[:n], nth)
    n1 = _size_for(f1, per, q.shape[0])
    nN = _size_for(fN, per, q.shape[0])
    out["o1_1thread"], _ = _best_rate(f1, n1)
    out["o1_all"], _ = _best_rate(fN, nN)
    out["o1_samples"] = [n1, nN]
    t0 = time.perf_counter()
    bpt = oracle.BPlusTree(fanout)
    bpt.insert_many(keys, vals)
    out["o2_build_s"] = time.perf_counter() - t0
    out["o2_height"] = bpt.height
    g1 = lambda n: bpt.search(q[:n], 1)
    gN = lambda n: bpt.search(q[:n], nth)
    m1 = _size_for(g1, per, q.shape[0])
    mN = _size_for(gN, per, q.shape[0])
    out["o2_1thread"], _ = _best_rate(g1, m1)
    out["o2_all"], _ = _best_rate(gN, mN)
    out["o2_samples"] = [m1, mN]
    return out


def run_reference(a, c, rank, world):
    """--impl reference: the CPU oracle (the only reference this paper-tier run has)."""
    if rank != 0:
        return
    T_ref = c["T"] // c.get("shards", 1)  # config 5: one shard (the CPU holds one shard's keys)
    keys = gen.uniform_keys(c["T"], count=T_ref) if T_ref != c["T"] else gen.uniform_keys(c["T"])
    vals = gen.values_for(keys)
    q = make_queries(keys, c["Q"], c["dist"], 0)
    import oracle

    nth = host_threads()
    # size one step so the whole run stays within a few minutes
    n = min(q.shape[0], 1 << 18)
    t0 = time.perf_counter()
    oracle.sorted_search(keys, vals, q[:n], nth)
    per_q = max(time.perf_counter() - t0, 1e-6) / n
    budget = 150.0 / max(1, a.steps + a.warmup)
    step_n = int(max(1 << 16, min(q.shape[0], budget / per_q)))
    for _ in range(a.warmup):
        oracle.sorted_search(keys, vals, q[:step_n], nth)
    t0 = time.perf_counter()
    for s in range(a.steps):
        off = (s * step_n) % max(1, q.shape[0] - step_n + 1)
        oracle.sorted_search(keys, vals, q[off:off + step_n], nth)
    dt = time.perf_counter() - t0
    v = step_n * a.steps / dt / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world,
        "steps": a.steps, "warmup": a.warmup, "ms_per_step": dt / a.steps * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64",
        "data": "synthetic", "config": {"workload": c["name"], "T": c["T"], "fanout": c["F"], "Q": c["Q"],
                                        "queries": c["dist"], "sample_per_step": step_n,
                                        "oracle_keys": int(T_ref)},
        "cpu_baseline": {"value": v, "unit": UNIT, "cores": nth, "kind": "oracle",
                         "sample": f"{step_n} of the {c['Q']} {c['dist']} queries per step; std::lower_bound "
                                   f"over {c['T']} sorted keys + value fetch, {nth} threads"},
        "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------ roofline
def roofline_model(info, plan, nq_window, l2_bytes):
    """Algorithmic bytes of the search kernel.

    Per launch over one PSA window of nw queries:
      I/O: 8 B query + position + 8 B result per query: the staged return reads a 2-B
           chunk-local offset (18 B), the other PSA paths a 4-B position (20 B), no PSA 16 B;
      tree: every level not staged in shared memory is charged min(no-reuse, whole level):
            no-reuse = nw x (S + 32) (node + one 32-B PS / value sector), whole level =
            nodes x S (+ the level's values for the leaf level).
    Returns (bytes_per_launch, no_reuse_bytes_per_query)."""
    F, h = info["fanout"], info["height"]
    S = F * 8
    ls = info["level_start"]
    io = (18 if plan.get("staged_return") else 20) if plan["psa_bits"] > 0 else 16
    tree = 0
    noreuse = io
    for lev in range(plan["smem_levels"], h):
        nodes = ls[lev + 1] - ls[lev]
        whole = nodes * S * (2 if lev == h - 1 else 1)
        tree += min(nq_window * (S + 32), whole)
        noreuse += S + 32
    return nq_window * io + tree, noreuse


def step_model(info, plan, nq, l2_cap, hbm_gbs, l2_gbs, psa=True):
    """Step-level roofline of SURVEY §8(d): bytes per query by tier and the bound
    min(BW_HBM / B_HBM, BW_L2 / B_L2) in G q/s.

    B_io = 16 (query in, result out), B_psa = 72 with PSA (histogram read 8, scatter 8 + 8 + 4,
    search 8 + 8, gather 4 + 32 + 8, minus B_io); every level below the shared-memory stage
    costs S + 32 (node + a PS or value sector).  Unstaged levels are in the L2 tier while their
    cumulative bytes (the leaf level with its values) stay within the L2 capacity (+5 %: the c2
    leaves + values are 131 MB against 126 MB, which SURVEY §8(d) counts as L2), the rest HBM.
    B_HBM = B_io + B_psa + HBM-tier levels; B_L2 = B_HBM + L2-tier levels (HBM bytes also pass
    L2).  The reuse-aware variant charges each tier min(no-reuse bytes, unique tier bytes / Q)."""
    F, h, ls = info["fanout"], info["height"], info["level_start"]
    S = F * 8
    b_io, b_psa = 16, (72 if psa else 0)
    cum, l2_lv, hbm_lv, l2_unique, hbm_unique = 0, 0, 0, 0, 0
    for lev in range(plan["smem_levels"], h):
        nodes = ls[lev + 1] - ls[lev]
        lbytes = nodes * S * (2 if lev == h - 1 else 1)
        cum += lbytes
        if cum <= 1.05 * l2_cap:
            l2_lv += S + 32
            l2_unique += lbytes
        else:
            hbm_lv += S + 32
            hbm_unique += lbytes
    b_hbm = b_io + b_psa + hbm_lv
    b_l2 = b_hbm + l2_lv
    bound = min(hbm_gbs / b_hbm, l2_gbs / b_l2)
    r_hbm = b_io + b_psa + min(hbm_lv, hbm_unique / nq)
    r_l2 = r_hbm + min(l2_lv, l2_unique / nq)
    rbound = min(hbm_gbs / r_hbm, l2_gbs / r_l2)
    return {"B_hbm": b_hbm, "B_l2": b_l2, "bound_gqs": bound, "l2_tier_levels": l2_lv // (S + 32),
            "hbm_tier_levels": hbm_lv // (S + 32),
            "reuse_aware": {"B_hbm": r_hbm, "B_l2": r_l2, "bound_gqs": rbound}}


def ncu_stats(workload, kernel, whole=False):
    """Per-launch ncu figures of `kernel` for `workload` from the committed capture summary
    (profiles/ncu_r2.json, tools/ncu_summary.py): DRAM and L2 bytes, sectors per request
    (the paper's memory divergence), warp coherence = active threads per
    executed instruction / 32 (P:L654 fn 4), branch uniformity."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "ncu_r2.json")))
        return d.get(workload, {}) if whole else d.get(workload, {}).get(kernel)
    except Exception:
        return None


STEP_KERNELS = ("k_psa2_rank", "k_psa2_move", "k_psa2_count_sort", "k_lane_search_c", "k_psa2_unmove")


def lsu_roofline(st, allk, nsm, mhz, avg_launch_ms, step_ms, one_level):
    """The search kernel's L1 data-pipe (LSU) roofline and the step's (DESIGN.md §7 item 4):
    every global / shared access, shared atomic and shuffle retires through the SM's L1 data
    pipe at one wavefront per cycle.  `st` / `allk`: per-launch ncu figures of the kernel and of
    every kernel of the workload (profiles/ncu_r2.json); nsm SMs at mhz (median SM clock in the
    timed region).  lsu = wavefronts per launch over the live launch time against nsm x clock;
    step_lsu (one-level staged path: the five kernels of a step, one launch each) = the
    LSU-bound step time against the measured one.  Returns (lsu, step_lsu), None when absent."""
    if not st or not st.get("lsu_wavefronts") or not mhz:
        return None, None
    lpeak = nsm * mhz * 1e6
    ach = st["lsu_wavefronts"] / (avg_launch_ms / 1e3)
    lsu = {"achieved": ach / 1e9, "peak": lpeak / 1e9, "unit": "G wavefronts/s", "frac": ach / lpeak,
           "wavefronts_per_launch": st["lsu_wavefronts"],
           "shared_wavefronts_per_launch": st.get("lsu_wavefronts_shared"),
           "peak_source": f"1 L1 data-pipe wavefront / cycle / SM x {nsm} SMs x {mhz:.0f} MHz "
                          "(median SM clock in the timed region)",
           "source": st.get("source")}
    step = None
    if one_level and all(allk.get(k, {}).get("lsu_wavefronts") for k in STEP_KERNELS):
        wsum = sum(allk[k]["lsu_wavefronts"] for k in STEP_KERNELS)
        bound_ms = wsum / lpeak * 1e3
        step = {"wavefronts_per_step": wsum, "bound_ms": bound_ms, "measured_ms": step_ms,
                "frac": bound_ms / step_ms, "kernels": list(STEP_KERNELS), "source": st.get("source")}
    return lsu, step


def load_peaks():
    hbm, src = 6650.0, "fallback (B200_PROFILING.md)"
    try:
        p = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
        hbm, src = float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        pass
    l2, l2src = None, None
    try:
        p = json.load(open(os.path.join(ROOT, "profiles", "r2_peaks.json")))
        l2, l2src = float(p["l2_read_gbs"]), "measured (profiles/r2_peaks.json, tools/peaks.cu)"
    except Exception:
        pass
    return hbm, src, l2, l2src


def timed(step, steps, stream):
    """K steps bracketed by CUDA events on the launch stream (one event pair per step):
    (total ms, per-step ms list)."""
    import torch

    ev = [torch.cuda.Event(enable_timing=True) for _ in range(steps + 1)]
    ev[0].record(stream)
    for i in range(steps):
        step()
        ev[i + 1].record(stream)
    torch.cuda.synchronize()
    per = [ev[i].elapsed_time(ev[i + 1]) for i in range(steps)]
    return ev[0].elapsed_time(ev[steps]), per


def run_extras(hm, dev, a):
    """Extra bench points measured in the default run: config 4 at N = 1 (the first point of
    the metric's 1/2/4/8-GPU curve) and config 3's fanout sweep (Zipf, theta 0.99).  Device-
    generated inputs; each point is warmed up and timed like the headline."""
    import torch

    out = {}
    stream = torch.cuda.current_stream(dev)

    def measure(t, q, steps):
        res = torch.empty_like(q)
        for _ in range(3):
            t.search(q, res)
        torch.cuda.synchronize()
        hm.profile_enable(True)
        hm.profile_read()
        ms, per = timed(lambda: t.search(q, res), steps, stream)
        hm.profile_enable(False)
        pr = hm.profile_read()
        ok = bool(torch.equal(res[:1 << 16].view(torch.int64), gen.values_for_t(q[:1 << 16].view(torch.int64))))
        return {"value": q.numel() / (ms / steps) / 1e6, "unit": UNIT, "ms_per_step": ms / steps,
                "ms_per_step_median": float(np.median(per)), "parity_sample_ok": ok,
                "kernels_ms_per_step": {k: v[0] / steps for k, v in pr.items()}}

    c4 = CONFIGS[4]
    keys = gen.uniform_keys_t(c4["T"], dev)
    t = hm.Tree(keys.view(torch.uint64), gen.values_for_t(keys).view(torch.uint64), fanout=c4["F"])
    q = gen.uniform_queries_t(keys, c4["Q"]).view(torch.uint64)
    r = measure(t, q, a.extra_steps)
    r.update({"workload": c4["name"] + "_n1", "plan": t.plan(c4["Q"])})
    out["c4_n1"] = r
    del t, q, keys
    torch.cuda.empty_cache()
    c3 = CONFIGS[3]
    keys = gen.uniform_keys_t(c3["T"], dev)
    qz = gen.zipf_queries_t(keys, c3["Q"]).view(torch.uint64)
    sweep = []
    for F in (8, 16, 32, 64, 128):
        t = hm.Tree(keys.view(torch.uint64), gen.values_for_t(keys).view(torch.uint64), fanout=F)
        r = measure(t, qz, max(3, a.extra_steps // 2))
        p = t.plan(c3["Q"])
        sweep.append({"fanout": F, "value": r["value"], "ms_per_step": r["ms_per_step"],
                      "parity_sample_ok": r["parity_sample_ok"], "psa_levels": p["psa_levels"],
                      "height": t.info()["height"]})
        del t
        torch.cuda.empty_cache()
    out["c3_fanout_sweep_zipf"] = {"workload": "c3_T2^26_Q2^26_zipf0.99", "unit": UNIT, "points": sweep}
    return out


def run_config5(a, c, hm, dev, world, rank, local, pg):
    """Config 5: key-range partitioned tree, one 2^29-key shard of the
    2^32-key set per rank (the 8-way partition; ranks 0..N-1 hold shards 0..N-1), queries
    uniform over the running ranks' keys routed by NCCL all-to-all (bypassed at N = 1), and
    one 2^22-op update batch (5 % insert, 5 % delete, 90 % update, routed) after every query
    batch.  value = queries of all ranks / max-over-ranks time of query + update
    batches; the update rate is reported beside it."""
    import torch

    from paper_conf_ppopp_yanlpz19_b200.dist import PartitionedTree

    T, P, S, F = c["T"], world, c["T"] // c["shards"], c["F"]
    if P > c["shards"]:
        raise SystemExit("config 5: at most %d ranks" % c["shards"])
    lk = gen.uniform_keys_t(T, dev, start=rank * S, count=S)
    sp = [int(x) & ((1 << 64) - 1) for x in gen.keys_at_t(T, torch.tensor([p * S for p in range(1, P)],
                                                                            dtype=torch.int64)).tolist()]
    t_build = time.perf_counter()
    pt = PartitionedTree(lk.view(torch.uint64), gen.values_for_t(lk).view(torch.uint64), sp, fanout=F,
                         fill=c.get("fill", 1.0), device=dev)
    torch.cuda.synchronize()
    t_build = time.perf_counter() - t_build
    del lk
    t = pt.ops.tree
    info = t.info()
    nidx = gen._t_umod(gen._t_stream(gen.SEED_QUERY, rank * c["Q"], c["Q"], dev), P * S)
    q = gen.keys_at_t(T, nidx).view(torch.uint64)
    del nidx
    nb = 8  # distinct update batches, cycled (each step applies a fresh batch of the cycle)
    batches = [gen.update_ops_t(T, c["ops"], 0.05, 0.05, dev, seed=gen.SEED_OPS + 1000 * b + rank, hi=P * S)
               for b in range(nb)]
    batches = [(o, k.view(torch.uint64), v.view(torch.uint64)) for o, k, v in batches]
    out = torch.empty_like(q)
    first = pt.search(q)
    torch.cuda.synchronize()
    sel = torch.from_numpy(np.asarray(gen._stream(99, 0, 1 << 16) % np.uint64(c["Q"]), dtype=np.int64)).to(dev)
    parity_ok = bool(torch.equal(first.view(torch.int64)[sel], gen.values_for_t(q.view(torch.int64)[sel])))
    it = [0]

    def step():
        out.copy_(pt.search(q))
        o, k, v = batches[it[0] % nb]
        it[0] += 1
        pt.update(o, k, v)

    for _ in range(max(3, a.warmup)):
        step()
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream(dev)
    if pg:
        pg.barrier()
    torch.cuda.synchronize()
    l0 = hm.kernel_launches()
    hm.profile_enable(True)
    hm.profile_read()
    with ClockSampler(local) as clk:
        ms, per_step = timed(step, a.steps, stream)
    hm.profile_enable(False)
    launches = hm.kernel_launches() - l0
    prof = hm.profile_read()
    ms_max = ms
    if pg:
        tt = torch.tensor([ms], device=dev, dtype=torch.float64)
        pg.all_reduce(tt, op=pg.ReduceOp.MAX)
        ms_max = float(tt.item())
    value = c["Q"] * world * a.steps / (ms_max / 1e3) / 1e9
    ups = c["ops"] * world * a.steps / (ms_max / 1e3) / 1e9
    e2e = None
    if not a.no_e2e:
        q_host = q.cpu().pin_memory()
        out_host = torch.empty(c["Q"], dtype=torch.uint64, pin_memory=True)
        # the host queries are written before the timed loop: the pipeline need not order its
        # first H2D copies after the previous step's work (HARMONIA_QF_HOST_UNORDERED)
        hopts = hm.make_opts(a.group_size, a.psa_bits, a.smem_levels, a.window, a.flags | hm.QF_HOST_UNORDERED)

        def e2e_step():
            pt.search_host(q_host, out_host, opts=hopts)
            o, k, v = batches[it[0] % nb]
            it[0] += 1
            pt.update(o, k, v)

        e2e_step()
        torch.cuda.synchronize()
        k2 = max(1, a.e2e_steps)
        hms, _ = timed(e2e_step, k2, stream)
        if pg:
            tt = torch.tensor([hms], device=dev, dtype=torch.float64)
            pg.all_reduce(tt, op=pg.ReduceOp.MAX)
            hms = float(tt.item())
        e2e = {"value": c["Q"] * world * k2 / (hms / 1e3) / 1e9, "unit": UNIT,
               "h2d_bytes_per_step": int(c["Q"] * 8), "d2h_bytes_per_step": int(c["Q"] * 8), "steps": k2,
               "ms_per_step": hms / k2, "api": "PartitionedTree.search_host + update (one shard: the tree's H2D/search/D2H pipeline; "
                      "several: pinned copies around the routed search)",
               "note": "update batches are device-resident (generated on the device) in both measurements"}
    if rank != 0:
        return
    hbm_peak, peak_src, _, _ = load_peaks()
    breakdown = {k: {"ms_per_step": v[0] / a.steps, "launches_per_step": v[1] / a.steps,
                     "share": v[0] / max(1e-9, sum(x[0] for x in prof.values()))} for k, v in prof.items()}
    roof = None
    dom = max(prof.items(), key=lambda kv: kv[1][0]) if prof else None
    mode = {1: "in place", 2: "full rebuild"}.get(t.last_update_mode(), "?")
    if dom and dom[0] == "update":
        avg = prof["update"][0] / prof["update"][1]
        if mode == "full rebuild":  # read records (16 B), write merged records (16 B), write the
            # key region + leaf values (16 B x F/(F-1)) per record of the shard
            byt = info["n_keys"] * (16 + 16 + 16 * F / (F - 1))
            what = "harmonia_update_batch (sort, merge, layout rebuild)"
        else:  # batch in (17 B/op) + key sort (2 x 12 B/op) + winners/locate/classify (~40 B/op)
            # + the changed leaves re-packed (2 x 1 KiB read + write per changed leaf, <= 1 per insert/delete)
            byt = c["ops"] * (17 + 24 + 40 + 0.1 * 2 * 2 * F * 8)
            what = "harmonia_update_batch in place (sort, locate, re-pack changed leaves)"
        roof = {"bound": "hbm", "kernel": what, "achieved": byt / (avg / 1e3) / 1e9, "peak": hbm_peak,
                "unit": "GB/s", "frac": byt / (avg / 1e3) / 1e9 / hbm_peak, "traffic": None,
                "peak_source": peak_src, "algorithmic_bytes_per_launch": byt, "avg_launch_ms": avg}
    elif dom and dom[0] == "search":
        avg = dom[1][0] / dom[1][1]
        plan5 = t.plan(c["Q"])
        byt, _ = roofline_model(info, plan5, c["Q"], 0)
        roof = {"bound": "hbm", "kernel": "k_lane_search_c", "achieved": byt / (avg / 1e3) / 1e9, "peak": hbm_peak,
                "unit": "GB/s", "frac": byt / (avg / 1e3) / 1e9 / hbm_peak, "traffic": None,
                "peak_source": peak_src, "algorithmic_bytes_per_launch": byt, "avg_launch_ms": avg}
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps,
        "warmup": max(3, a.warmup), "ms_per_step": ms_max / a.steps,
        "ms_per_step_median": float(np.median(per_step)), "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u64", "data": "synthetic",
        "config": {"workload": c["name"], "T": T, "shard_keys": S, "fanout": F, "Q_per_gpu": c["Q"],
                   "update_ops_per_step_per_gpu": c["ops"], "update_mix": "5% insert, 5% delete, 90% update",
                   "queries": "uniform over the running shards' keys", "mode": "partitioned",
                   "l2_flush": "inputs_larger_than_L2 (2^27 queries + a 2^29-key shard per GPU)",
                   "plan": t.plan(c["Q"]), "height": info["height"], "build_s": t_build},
        "updates_per_s": {"value": ups, "unit": "G ops/s", "mode": mode},
        "roofline": roof, "cpu_baseline": None, "e2e": e2e, "gpu_launches": int(launches),
        "clocks": clk.summary(), "kernel_breakdown": breakdown, "parity_sample_ok": parity_ok,
    }
    print(json.dumps(line), flush=True)


def main():
    a = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    c = workload(a)

    if a.impl == "reference":
        if world > 1:
            import torch.distributed as dist

            dist.init_process_group("gloo")
            run_reference(a, c, rank, world)
            dist.barrier()
            dist.destroy_process_group()
        else:
            run_reference(a, c, rank, world)
        return

    import torch

    import paper_conf_ppopp_yanlpz19_b200 as hm

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    pg = None
    if world > 1 or a.mode in ("partitioned", "peer") or a.config == 5:
        import torch.distributed as dist

        if world == 1:  # a one-rank group without torchrun (--mode partitioned/peer at N = 1)
            os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
            os.environ.setdefault("MASTER_PORT", str(29500 + os.getpid() % 1000))
            os.environ.setdefault("RANK", "0")
            os.environ.setdefault("WORLD_SIZE", "1")
        # NCCL prints its version banner on the C-level stdout at communicator creation; route
        # fd 1 to stderr meanwhile so stdout carries only the JSON line
        sys.stdout.flush()
        saved = os.dup(1)
        os.dup2(2, 1)
        try:
            dist.init_process_group("nccl", device_id=dev)
            dist.barrier()
            torch.cuda.synchronize()
        finally:
            sys.stdout.flush()
            os.dup2(saved, 1)
            os.close(saved)
        pg = dist

    def barrier():
        if pg:
            pg.barrier()

    if a.config == 5:
        run_config5(a, c, hm, dev, world, rank, local, pg)
        if pg:
            pg.destroy_process_group()
        return

    # ---- inputs (synthetic, seeded).  replicated: identical tree on every rank, each rank its
    # own slice of the global query stream (weak scaling, no collective).  partitioned: rank p
    # holds the key-quantile shard p; its queries are uniform over the global key set and are
    # routed to their shards by NCCL all-to-all (the real exchange step).
    keys = gen.uniform_keys(c["T"])
    vals = gen.values_for(keys)
    opts = hm.make_opts(a.group_size, a.psa_bits, a.smem_levels, a.window, a.flags)
    pt = None
    if a.mode in ("partitioned", "peer"):
        from paper_conf_ppopp_yanlpz19_b200.dist import PartitionedTree, PeerPartitionedTree, key_splitters

        sp = key_splitters(keys, world)
        bnd = [0] + [int(np.searchsorted(keys, np.uint64(s))) for s in sp] + [c["T"]]
        lk, lv = keys[bnd[rank]:bnd[rank + 1]], vals[bnd[rank]:bnd[rank + 1]]
        cls = PeerPartitionedTree if a.mode == "peer" else PartitionedTree
        pt = cls(torch.from_numpy(lk).to(dev), torch.from_numpy(lv).to(dev), sp, fanout=c["F"], fill=a.fill,
                 device=dev)
        t = pt.ops.tree
    elif world > 1:  # replicated mode: the same layout on every rank, no collective on the hot path
        from paper_conf_ppopp_yanlpz19_b200.dist import ReplicatedTree

        t = ReplicatedTree(torch.from_numpy(keys).to(dev), torch.from_numpy(vals).to(dev), fanout=c["F"],
                           fill=a.fill).tree
    else:
        t = hm.Tree(torch.from_numpy(keys).to(dev), torch.from_numpy(vals).to(dev), fanout=c["F"], fill=a.fill)
    info = t.info()
    q_np = make_queries(keys, c["Q"], c["dist"], rank)
    q_host = torch.from_numpy(q_np).pin_memory()
    q = q_host.to(dev)
    out = torch.empty_like(q)
    plan = t.plan(c["Q"], opts)

    def step():
        if pt is not None:
            out.copy_(pt.search(q, slices=a.slices) if a.mode == "partitioned" else pt.search(q))
        else:
            t.search(q, out, opts=opts)

    if a.sweep:
        for spec in a.sweep.split(";"):
            kw = dict(group_size=a.group_size, psa_bits=a.psa_bits, smem_levels=a.smem_levels, window=a.window,
                      flags=a.flags, lane_queries=0)
            for item in filter(None, spec.split(",")):
                k, v = item.split("=")
                kw[k] = int(v)
            o = hm.make_opts(**kw)
            for _ in range(3):
                t.search(q, out, opts=o)
            torch.cuda.synchronize()
            s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            hm.profile_enable(True)
            hm.profile_read()
            s0.record()
            for _ in range(a.steps):
                t.search(q, out, opts=o)
            s1.record()
            torch.cuda.synchronize()
            hm.profile_enable(False)
            pr = hm.profile_read()
            ms_ = s0.elapsed_time(s1) / a.steps
            print(json.dumps({"sweep": kw, "gqs": c["Q"] / ms_ / 1e6, "ms": ms_, "plan": t.plan(c["Q"], o),
                              "kernels_ms_per_step": {k: v[0] / a.steps for k, v in pr.items()}}), flush=True)
        return

    for _ in range(max(3, a.warmup)):
        step()
    torch.cuda.synchronize()
    # property check on this rank's batch: values are key-derived (uniform/zipf hit 100 %)
    sel = np.asarray(gen._stream(99, 0, 1 << 16) % np.uint64(c["Q"]), dtype=np.int64)
    got = out.view(torch.int64)[torch.from_numpy(sel).to(dev)].cpu().numpy().view(np.uint64)
    parity_ok = bool(np.array_equal(got, gen.values_for(q_np[sel])))

    # ---- timed region: K steps, events on the launch stream, max over ranks
    stream = torch.cuda.current_stream(dev)
    barrier()
    torch.cuda.synchronize()
    l0 = hm.kernel_launches()
    hm.profile_enable(True)
    hm.profile_read()
    with ClockSampler(local) as clk:
        ms, per_step = timed(step, a.steps, stream)
    hm.profile_enable(False)
    launches = hm.kernel_launches() - l0
    prof = hm.profile_read()
    barrier()
    ms_max = ms
    if pg:
        tt = torch.tensor([ms], device=dev, dtype=torch.float64)
        pg.all_reduce(tt, op=pg.ReduceOp.MAX)
        ms_max = float(tt.item())
    total_q = c["Q"] * world * a.steps
    value = total_q / (ms_max / 1e3) / 1e9

    # ---- end to end through the public API with host buffers
    e2e = None
    if not a.no_e2e:
        out_host = torch.empty(c["Q"], dtype=torch.uint64, pin_memory=True)
        # the host queries are written before the timed loop: the pipeline need not order its
        # first H2D copies after the previous step's work (HARMONIA_QF_HOST_UNORDERED)
        hopts = hm.make_opts(a.group_size, a.psa_bits, a.smem_levels, a.window, a.flags | hm.QF_HOST_UNORDERED)

        def e2e_step():
            if pt is not None:  # H2D, routed search, D2H through the same public objects
                q.copy_(q_host, non_blocking=True)
                out_host.copy_(pt.search(q), non_blocking=True)
            else:
                t.search_host(q_host, out_host, opts=hopts)

        e2e_step()
        torch.cuda.synchronize()
        barrier()
        torch.cuda.synchronize()
        h0, h1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        k2 = max(1, a.e2e_steps)
        h0.record(stream)
        for _ in range(k2):
            e2e_step()
        h1.record(stream)
        torch.cuda.synchronize()
        hms = h0.elapsed_time(h1)
        if pg:
            tt = torch.tensor([hms], device=dev, dtype=torch.float64)
            pg.all_reduce(tt, op=pg.ReduceOp.MAX)
            hms = float(tt.item())
        e2e_ok = bool(np.array_equal(out_host.numpy()[sel], gen.values_for(q_np[sel])))
        parity_ok = parity_ok and e2e_ok
        e2e = {"value": c["Q"] * world * k2 / (hms / 1e3) / 1e9, "unit": UNIT,
               "h2d_bytes_per_step": int(c["Q"] * 8), "d2h_bytes_per_step": int(c["Q"] * 8),
               "steps": k2, "ms_per_step": hms / k2,
               "api": type(pt).__name__ + ".search + pinned copies" if pt is not None else
               "harmonia_search_batch_host (pinned)"}

    if rank != 0:
        if pg:
            pg.destroy_process_group()
        return

    # ---- roofline of the dominant kernel (events around each launch, same stream)
    hbm_peak, peak_src, l2_peak, l2_src = load_peaks()
    dom = max(prof.items(), key=lambda kv: kv[1][0]) if prof else ("search", (ms, 1))
    dom_kind, (dom_ms, dom_n) = dom
    l2_bytes = torch.cuda.get_device_properties(dev).L2_cache_size
    nw = plan["window"] if plan["window"] else c["Q"]
    bytes_launch, noreuse_bpq = roofline_model(info, plan, nw, l2_bytes)
    # profiling classes of the C ABI -> the kernels they time on the default staged-return path
    kernels = {"search": "k_lane_search_c (Eq-1 descent + leaf probe, results to level-1 order)",
               "psa_hist": "k_psa2_rank (level-1 digit + rank in tile)",
               "psa_scatter": "k_psa2_move (level-1 staged move)",
               "psa_scan": "k_psa2_count_sort (level-2 chunk counting sort)",
               "return": "k_psa2_unmove (inverse move to caller order)"}
    breakdown = {k: {"ms_per_step": v[0] / a.steps, "launches_per_step": v[1] / a.steps,
                     "share": v[0] / max(1e-9, sum(x[0] for x in prof.values())),
                     "kernels": kernels.get(k, k)} for k, v in prof.items()}
    roof = None
    if dom_kind == "search":
        avg_ms = dom_ms / dom_n
        achieved = bytes_launch / (avg_ms / 1e3) / 1e9
        kname = ("k_lane_search_c" if plan.get("staged_return") else "k_lane_search_u") \
            if plan["group_size"] == 1 else "k_ntg_search2"
        roof = {"bound": "hbm", "kernel": kname, "achieved": achieved, "peak": hbm_peak,
                "unit": "GB/s", "frac": achieved / hbm_peak, "traffic": None, "peak_source": peak_src,
                "algorithmic_bytes_per_launch": bytes_launch, "queries_per_launch": nw,
                "avg_launch_ms": avg_ms, "no_reuse_bytes_per_query": noreuse_bpq,
                "no_reuse_frac": (nw * noreuse_bpq) / (avg_ms / 1e3) / 1e9 / hbm_peak}
    else:
        # PSA kernels are streaming passes over the window: 8 B read (+12 B written by scatter)
        # rank: 8 B query in, 4 B packed digit/rank out; move: query + packed in, query out;
        # chunk sort: query in, query + 4 B offset out; unmove: packed + result in, result out
        per_q = {"psa_hist": 8 + 4, "psa_scatter": 8 + 4 + 8, "psa_scan": 8 + 8 + 4,
                 "return": 4 + 8 + 8}.get(dom_kind, 8)
        avg_ms = dom_ms / dom_n
        achieved = nw * per_q / (avg_ms / 1e3) / 1e9
        roof = {"bound": "hbm", "kernel": dom_kind, "achieved": achieved, "peak": hbm_peak, "unit": "GB/s",
                "frac": achieved / hbm_peak, "traffic": None, "peak_source": peak_src,
                "algorithmic_bytes_per_launch": nw * per_q, "avg_launch_ms": avg_ms}
    # L2 tier of the same kernel: its L2 traffic per launch (ncu lts__t_bytes of the committed
    # capture) over the live launch time, against the measured L2 read peak; and the step-level
    # model of SURVEY §8(d) (no-reuse and reuse-aware) against the measured step rate
    st = ncu_stats(c["name"], roof["kernel"]) if roof else None
    if roof is not None and st:
        roof["traffic"] = st.get("dram_bytes")
        roof["traffic_source"] = st.get("source")
        if l2_peak and st.get("lts_bytes"):
            ach = st["lts_bytes"] / (roof["avg_launch_ms"] / 1e3) / 1e9
            roof["l2"] = {"achieved": ach, "peak": l2_peak, "unit": "GB/s", "frac": ach / l2_peak,
                          "bytes_per_launch": st["lts_bytes"], "peak_source": l2_src,
                          "bytes_source": st.get("source")}
        roof["ncu"] = {k: st[k] for k in ("sectors_per_request", "warp_coherence", "branch_uniform_pct",
                                          "dram_bytes_per_query", "lts_bytes_per_query", "l1_hit_pct",
                                          "lts_hit_pct", "issue_active_pct", "l1_wavefront_pct", "lts_pct",
                                          "long_scoreboard_stall_share") if k in st}
        if "l1_wavefront_pct" in st:  # the on-chip limiter of the search
            roof["limiter"] = {"resource": "L1 data-pipe (LSU) wavefronts", "frac": st["l1_wavefront_pct"] / 100,
                               "source": st.get("source")}
        # the same limiter as a roofline on the live launch time: the kernel's LSU wavefronts
        # per launch (committed capture) against 1 wavefront per cycle per SM at the median SM
        # clock sampled during the timed region; and for the whole step (every kernel of the
        # step, one launch each), the LSU-bound step time against the measured one
        mhz = clk.summary().get("sm_mhz")
        nsm = torch.cuda.get_device_properties(dev).multi_processor_count
        one_level = bool(plan.get("staged_return")) and plan.get("psa_levels") == 1
        lsu, step_lsu = lsu_roofline(st, ncu_stats(c["name"], None, whole=True) or {}, nsm, mhz,
                                     roof["avg_launch_ms"], ms_max / a.steps, one_level)
        if lsu:
            roof["lsu"] = lsu
        if step_lsu:
            roof["step_lsu"] = step_lsu
    if roof is not None and l2_peak:
        sm_ = step_model(info, plan, c["Q"] * 1, l2_bytes, hbm_peak, l2_peak, psa=plan["psa_bits"] > 0)
        sm_["frac"] = value / world / sm_["bound_gqs"]
        sm_["reuse_aware"]["frac"] = value / world / sm_["reuse_aware"]["bound_gqs"]
        sm_["note"] = "per GPU; no-reuse frac > 1 means PSA neighbours share nodes (SURVEY §8(d) caveat)"
        roof["step_model"] = sm_

    cpu = None
    if not a.no_cpu and world == 1:
        cb = cpu_baselines(keys, vals, q_np, a.cpu_seconds, c["F"])
        cpu = {"value": cb["o1_all"] / 1e9, "unit": UNIT, "cores": cb["cores"], "kind": "oracle",
               "sample": f"prefixes of the {c['Q']} {c['dist']} queries ({cb['o1_samples'][1]} for all threads, "
                         f"{cb['o1_samples'][0]} for 1 thread); std::lower_bound over {c['T']} sorted keys + value "
                         f"fetch; best of 5 after 1 warm-up", "cpu_model": cb["cpu_model"],
               "one_thread": cb["o1_1thread"] / 1e9,
               "bptree": {"value": cb["o2_all"] / 1e9, "one_thread": cb["o2_1thread"] / 1e9,
                          "what": f"O2 pointer B+tree (P:L120/L218), fanout {c['F']}, built by sorted insertion "
                                  f"in {cb['o2_build_s']:.1f} s, height {cb['o2_height']}",
                          "samples": cb["o2_samples"]}}
    extra = None
    if a.config == 2 and world == 1 and not a.no_extra and not (a.keys or a.queries or a.fanout or a.dist):
        del q, out
        torch.cuda.empty_cache()
        extra = run_extras(hm, dev, a)

    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps,
        "warmup": max(3, a.warmup), "ms_per_step": ms_max / a.steps,
        "ms_per_step_median": float(np.median(per_step)), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
        "config": {"workload": c["name"], "T": c["T"], "fanout": c["F"], "fill": a.fill, "Q_per_gpu": c["Q"],
                   "queries": c["dist"], "mode": a.mode if (world > 1 or a.mode in ("partitioned", "peer")) else "single",
                   "l2_flush": "inputs_larger_than_L2 (queries+results %d MiB/GPU > L2 %d MiB)" % (
                       c["Q"] * 16 >> 20, l2_bytes >> 20),
                   "plan": plan, "height": info["height"]},
        "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": int(launches),
        "clocks": clk.summary(), "kernel_breakdown": breakdown, "parity_sample_ok": parity_ok,
        "context": {"paper_titan_v_gqs": PAPER_TITANV_GQS, "note": "P:L40/L592, TITAN V — other hardware"},
    }
    if extra:
        line["extra"] = extra
    print(json.dumps(line), flush=True)
    if pg:
        pg.destroy_process_group()


if __name__ == "__main__":
    main()
