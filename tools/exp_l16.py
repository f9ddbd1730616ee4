"""Measurement helper: one vs two PSA levels (harmonia_plan.psa_levels) per config, per kernel
class (CUDA events), device-resident batches.  Usage: python tools/exp_l16.py [cfg ...]
with cfg in c2, c3u, c3z, c4, t24, t25."""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import harmonia_gen as gen  # noqa: E402
import paper_conf_ppopp_yanlpz19_b200 as hm  # noqa: E402

CFG = {"c2": (23, 26, "uniform"), "c3u": (26, 26, "uniform"), "c3z": (26, 26, "zipf"), "c4": (28, 27, "uniform"),
       "t24": (24, 26, "uniform"), "t25": (25, 26, "uniform")}


def run(name, variants, reps=5):
    lt, lq, dist = CFG[name]
    keys = gen.uniform_keys_t(1 << lt, "cuda")
    t = hm.Tree(keys.view(torch.uint64), gen.values_for_t(keys).view(torch.uint64), fanout=64)
    if dist == "zipf":
        q = torch.from_numpy(gen.zipf_queries(keys.cpu().numpy().view(np.uint64), 1 << lq).view(np.int64)).cuda()
    else:
        q = gen.uniform_queries_t(keys, 1 << lq)
    q = q.view(torch.uint64)
    for vname, kw in variants:
        out = t.search(q, **kw)
        torch.cuda.synchronize()
        ok = bool(torch.equal(out.view(torch.int64), gen.values_for_t(q.view(torch.int64))))
        t.search(q, **kw)
        torch.cuda.synchronize()
        hm.profile_enable(True)
        hm.profile_read()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            t.search(q, out=out, **kw)
        e1.record()
        torch.cuda.synchronize()
        r = hm.profile_read()
        hm.profile_enable(False)
        ms = e0.elapsed_time(e1) / reps
        plan = t.plan(1 << lq, **kw)
        print(name, vname, f"levels={plan['psa_levels']} chunk={plan['sort_chunk']} K={plan['chunk_group']}",
              f"{ms:.3f} ms  {(1 << lq) / ms / 1e6:.2f} Gq/s ok={ok}",
              {k: round(v[0] / reps, 3) for k, v in r.items() if v[0]}, flush=True)
    del t, q, keys
    torch.cuda.empty_cache()


if __name__ == "__main__":
    names = sys.argv[1:] or ["c2", "c3u", "c4"]
    V = [("L8", dict(flags=hm.QF_PSA_L8)), ("L16c4k", dict(flags=hm.QF_PSA_L16, sort_chunk=4096)),
         ("L16c8k", dict(flags=hm.QF_PSA_L16, sort_chunk=8192)), ("auto", {})]
    for n in names:
        t0 = time.time()
        run(n, V)
        print("#", n, f"{time.time() - t0:.1f}s", flush=True)
