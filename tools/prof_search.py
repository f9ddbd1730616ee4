"""Small driver for ncu captures: build a config-2 tree (or --keys/--fanout) and run a few
harmonia_search_batch calls with the given options.  Never used for bench numbers."""
import argparse
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import harmonia_gen as gen  # noqa: E402
import paper_conf_ppopp_yanlpz19_b200 as hm  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--keys", type=int, default=23)
ap.add_argument("--queries", type=int, default=26)
ap.add_argument("--fanout", type=int, default=64)
ap.add_argument("--dist", default="uniform")
ap.add_argument("--calls", type=int, default=3)
ap.add_argument("--group-size", type=int, default=0)
ap.add_argument("--psa-bits", type=int, default=0)
ap.add_argument("--window", type=int, default=0)
ap.add_argument("--smem-levels", type=int, default=0)
ap.add_argument("--flags", type=int, default=0)
ap.add_argument("--range-len", type=int, default=0)
a = ap.parse_args()

kt = gen.uniform_keys_t(1 << a.keys, "cuda")  # device generators (= the numpy streams, tests/test_gen.py)
t = hm.Tree(kt.view(torch.uint64), gen.values_for_t(kt).view(torch.uint64), fanout=a.fanout)
o = hm.make_opts(a.group_size, a.psa_bits, a.smem_levels, a.window, a.flags)
if a.range_len:
    keys = kt.cpu().numpy().view(np.uint64)
    lo, hi = gen.ranges(keys, 1 << a.queries, a.range_len)
    lo, hi = torch.from_numpy(lo).cuda(), torch.from_numpy(hi).cuda()
    for _ in range(a.calls):
        t.range(lo, hi, a.range_len, opts=o)
else:
    q = gen.zipf_queries_t(kt, 1 << a.queries) if a.dist == "zipf" else gen.uniform_queries_t(kt, 1 << a.queries)
    q = q.view(torch.uint64)
    out = torch.empty_like(q)
    for _ in range(a.calls):
        t.search(q, out, opts=o)
torch.cuda.synchronize()
print("plan", t.plan(1 << a.queries, o))
