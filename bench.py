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
def cpu_oracle_rate(keys, vals, q, seconds):
    """Time the oracle (std::lower_bound, all host threads) on a bounded sample of q."""
    import oracle

    nth = host_threads()
    n = min(q.shape[0], 1 << 18)
    t0 = time.perf_counter()
    oracle.sorted_search(keys, vals, q[:n], nth)
    dt = max(time.perf_counter() - t0, 1e-6)
    n2 = int(min(q.shape[0], max(n, n * seconds / dt)))
    t0 = time.perf_counter()
    oracle.sorted_search(keys, vals, q[:n2], nth)
    dt2 = time.perf_counter() - t0
    return n2, dt2, nth


def run_reference(a, c, rank, world):
    """--impl reference: the CPU oracle (the only reference this paper-tier run has)."""
    if rank != 0:
        return
    keys = gen.uniform_keys(c["T"])
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
                                        "queries": c["dist"], "sample_per_step": step_n},
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
    if world > 1 or a.mode in ("partitioned", "peer"):
        import torch.distributed as dist

        if world == 1:  # a one-rank group without torchrun (--mode partitioned/peer at N = 1)
            os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
            os.environ.setdefault("MASTER_PORT", str(29500 + os.getpid() % 1000))
            os.environ.setdefault("RANK", "0")
            os.environ.setdefault("WORLD_SIZE", "1")
        dist.init_process_group("nccl", device_id=dev)
        pg = dist

    def barrier():
        if pg:
            pg.barrier()

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
            out.copy_(pt.search(q))
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
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    torch.cuda.synchronize()
    l0 = hm.kernel_launches()
    hm.profile_enable(True)
    hm.profile_read()
    with ClockSampler(local) as clk:
        e0.record(stream)
        for _ in range(a.steps):
            step()
        e1.record(stream)
        torch.cuda.synchronize()
    hm.profile_enable(False)
    launches = hm.kernel_launches() - l0
    prof = hm.profile_read()
    barrier()
    ms = e0.elapsed_time(e1)
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

        def e2e_step():
            if pt is not None:  # H2D, routed search, D2H through the same public objects
                q.copy_(q_host, non_blocking=True)
                out_host.copy_(pt.search(q), non_blocking=True)
            else:
                t.search_host(q_host, out_host, opts=opts)

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
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
        hbm_peak, peak_src = float(peaks["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        hbm_peak, peak_src = 6650.0, "fallback (B200_PROFILING.md)"
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
    # ncu DRAM traffic per launch, if a capture summary was committed for this workload
    try:
        prof_sum = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))
        ent = prof_sum.get(c["name"], {}).get(roof["kernel"])
        if ent:
            roof["traffic"] = ent["dram_bytes_per_launch"]
            roof["traffic_source"] = ent.get("source")
            if "l1_wavefront_pct" in ent:  # the on-chip limiter of the search
                roof["limiter"] = {"resource": "L1 data-pipe (LSU) wavefronts", "frac": ent["l1_wavefront_pct"] / 100,
                                   "source": ent.get("source")}
            if ent.get("sol_pct"):  # ncu speed-of-light of every tier: none saturated -> latency-bound
                roof["ncu_sol"] = {k: v / 100 for k, v in ent["sol_pct"].items()}
                if ent.get("ncu_time_s"):  # DRAM GB/s of the captured launch vs the measured peak
                    roof["ncu_sol"]["dram"] = ent["dram_bytes_per_launch"] / ent["ncu_time_s"] / 1e9 / hbm_peak
                if "long_scoreboard_stall_share" in ent:
                    roof["ncu_sol"]["long_scoreboard_stall_share"] = ent["long_scoreboard_stall_share"]
    except Exception:
        pass

    cpu = None
    if not a.no_cpu and world == 1:
        n2, dt2, nth = cpu_oracle_rate(keys, vals, q_np, a.cpu_seconds)
        cpu = {"value": n2 / dt2 / 1e9, "unit": UNIT, "cores": nth, "kind": "oracle",
               "sample": f"first {n2} of the {c['Q']} {c['dist']} queries; std::lower_bound over {c['T']} "
                         f"sorted keys + value fetch; {dt2:.1f} s"}

    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps,
        "warmup": max(3, a.warmup), "ms_per_step": ms_max / a.steps, "higher_is_better": True,
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
    print(json.dumps(line), flush=True)
    if pg:
        pg.destroy_process_group()


if __name__ == "__main__":
    main()
