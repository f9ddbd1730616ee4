"""Secondary measurements (not the contract line): update throughput (P:L546 mix), range
throughput (config-4 lengths on one GPU), and the config-3 fanout x G sweep.

  python tools/bench_extras.py [--what update,range,sweep] > profiles/rNN_extras.jsonl
Each measurement prints one JSON line; CUDA-event timing on the launch stream after warm-up.
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import harmonia_gen as gen  # noqa: E402
import paper_conf_ppopp_yanlpz19_b200 as hm  # noqa: E402


def timed(fn, reps, warm=2):
    # two warm-up calls: an update batch alternates the live and spare layout buffers, so the
    # second call is the one that grows the spare set after the first call grew the tree
    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    s0.record()
    for _ in range(reps):
        fn()
    s1.record()
    torch.cuda.synchronize()
    return s0.elapsed_time(s1) / reps


def update_bench(T=1 << 23, batch=1 << 22, reps=3):
    """4M-op batches (P:L546 mixes) on a fill-1.0 tree (every leaf full: inserts force the
    full rebuild) and on a fill-0.69 tree (the paper's insertion-built occupancy: in place)."""
    keys = gen.uniform_keys(T)
    vals = gen.values_for(keys)
    res = []
    for fill in (1.0, 0.69):
        t = hm.Tree(torch.from_numpy(keys).cuda(), torch.from_numpy(vals).cuda(), fanout=64, fill=fill)
        for ins, dele in ((0.05, 0.0), (0.05, 0.05)):
            ops, ks, vs = gen.update_ops(keys, batch, insert_frac=ins, delete_frac=dele)
            o, k, v = torch.from_numpy(ops).cuda(), torch.from_numpy(ks).cuda(), torch.from_numpy(vs).cuda()
            ms = timed(lambda: t.update(o, k, v), reps)
            mode = {1: "in place", 2: "full rebuild"}.get(t.last_update_mode(), "?")
            res.append({"what": "update_batch", "T": T, "fill": fill, "batch": batch, "insert": ins, "delete": dele,
                        "ms_per_batch": ms, "Mops_per_s": batch / ms / 1e3, "mode": mode,
                        "note": "device-resident batch; sort, winners, then " + mode})
            print(json.dumps(res[-1]), flush=True)
        del t
    return []


def range_bench(T=1 << 23, F=64, reps=5, groups=(0,), flags=0):
    keys = gen.uniform_keys(T)
    vals = gen.values_for(keys)
    t = hm.Tree(torch.from_numpy(keys).cuda(), torch.from_numpy(vals).cuda(), fanout=F)
    res = []
    for length, Qr in ((16, 1 << 22), (64, 1 << 21), (256, 1 << 20), (1024, 1 << 18)):
        lo, hi = gen.ranges(keys, Qr, length)
        lo, hi = torch.from_numpy(lo).cuda(), torch.from_numpy(hi).cuda()
        outb = (torch.empty((Qr, length), dtype=torch.uint64, device="cuda"),
                torch.empty((Qr, length), dtype=torch.uint64, device="cuda"),
                torch.empty(Qr, dtype=torch.uint32, device="cuda"))
        for G in groups:
            o = hm.make_opts(group_size=G, flags=flags)
            ms = timed(lambda: t.range(lo, hi, length, out=outb, opts=o), reps)  # slabs preallocated
            cnt = outb[2].cpu().numpy()
            ok = bool((cnt == length).all())  # lo = key[p], hi = key[p+len-1]: exactly len records
            res.append({"what": "range_batch", "T": T, "F": F, "G": G, "len": length, "Qr": Qr, "ms": ms,
                        "kernel": ("group" if (G or flags & (hm.QF_RANGE_GROUP | hm.QF_NO_RANGE_LANE)) else
                                   ("lane" if length < 512 else "warp")), "counts_ok": ok,
                        "Gq_per_s": Qr / ms / 1e6, "G_records_per_s": Qr * length / ms / 1e6,
                        "GB_per_s_out": Qr * length * 16 / ms / 1e6})
            print(json.dumps(res[-1]), flush=True)
    return []


def sweep_bench(T=1 << 26, Q=1 << 26, dist="zipf", reps=5):
    keys = gen.uniform_keys(T)
    vals = gen.values_for(keys)
    q = gen.zipf_queries(keys, Q) if dist == "zipf" else gen.uniform_queries(keys, Q)
    qd = torch.from_numpy(q).cuda()
    out = torch.empty_like(qd)
    res = []
    for F in (8, 16, 32, 64, 128):
        t = hm.Tree(torch.from_numpy(keys).cuda(), torch.from_numpy(vals).cuda(), fanout=F)
        for G in (2, 4, 8, 16, 32):
            if 2 * G > F:
                continue
            for flags in (0, hm.QF_LINEAR):
                o = hm.make_opts(group_size=G, flags=flags)
                ms = timed(lambda: t.search(qd, out, opts=o), reps)
                res.append({"what": "search_sweep", "T": T, "Q": Q, "dist": dist, "F": F, "G": G,
                            "node_search": "linear" if flags else "kary", "ms": ms, "Gq_per_s": Q / ms / 1e6,
                            "height": t.info()["height"]})
                print(json.dumps(res[-1]), flush=True)
        t.close()
        torch.cuda.empty_cache()
    return []


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--what", default="update,range")
    ap.add_argument("--sweep-dist", default="zipf")
    a = ap.parse_args()
    for w in a.what.split(","):
        rows = {"update": update_bench, "range": range_bench,
                "range_sweep": lambda: range_bench(groups=(2, 4, 8, 16, 32)),
                "range_group": lambda: range_bench(flags=hm.QF_RANGE_GROUP),
                "range_nolane": lambda: range_bench(flags=hm.QF_NO_RANGE_LANE),
                "sweep": lambda: sweep_bench(dist=a.sweep_dist)}[w]()
        for r in rows:
            print(json.dumps(r), flush=True)
