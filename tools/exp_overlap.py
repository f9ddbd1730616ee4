"""Experiment: does splitting the batch into sub-batches on two streams (so one sub-batch's
PSA passes run beside the other's search) raise c2 throughput?  Measurement only.

    HARMONIA_LIB=tools/bin/<variant>.so python tools/exp_overlap.py [tag] [--chunk 4096]
"""
import argparse
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import harmonia_gen as gen  # noqa: E402
import paper_conf_ppopp_yanlpz19_b200 as hm  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("tag", nargs="?", default="?")
ap.add_argument("--keys", type=int, default=23)
ap.add_argument("--queries", type=int, default=26)
ap.add_argument("--chunk", type=int, default=0)
ap.add_argument("--parts", type=int, default=2)
ap.add_argument("--streams", type=int, default=2)
args = ap.parse_args()

keys = gen.uniform_keys_t(1 << args.keys, "cuda")
t = hm.Tree(keys.view(torch.uint64), gen.values_for_t(keys).view(torch.uint64), fanout=64)
q = gen.uniform_queries_t(keys, 1 << args.queries).view(torch.uint64)
out = torch.empty_like(q)
n = q.numel()
streams = [torch.cuda.current_stream()] + [torch.cuda.Stream() for _ in range(args.streams - 1)]
ev_done = [torch.cuda.Event() for _ in streams]
kw = {"sort_chunk": args.chunk} if args.chunk else {}


def step_single():
    t.search(q, out, **kw)


def step_split():
    cur = torch.cuda.current_stream()
    start = torch.cuda.Event()
    start.record(cur)
    P = args.parts
    for i in range(P):
        s = streams[i % len(streams)]
        s.wait_event(start)
        a, b = i * n // P, (i + 1) * n // P
        t.search(q[a:b], out[a:b], stream=s, **kw)
    for j, s in enumerate(streams):
        ev_done[j].record(s)
        cur.wait_event(ev_done[j])


def timeit(fn, reps=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    best = 1e9
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            fn()
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1) / reps)
    return best


ref = gen.values_for_t(q.view(torch.int64)).view(torch.uint64)
ms1 = timeit(step_single)
ok1 = bool(torch.equal(out, ref))
out.zero_()
ms2 = timeit(step_split)
ok2 = bool(torch.equal(out, ref))
print(args.tag, f"T=2^{args.keys} Q=2^{args.queries} chunk={args.chunk or 'auto'}",
      f"single {ms1:.3f} ms {n / ms1 / 1e6:.2f} Gq/s ok={ok1} |",
      f"split{args.parts}x{args.streams}st {ms2:.3f} ms {n / ms2 / 1e6:.2f} Gq/s ok={ok2}", flush=True)
