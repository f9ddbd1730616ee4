"""A/B helper: c2 (or --keys) step and kernel times for the library found by the import path
(HARMONIA_LIB / PYTHONPATH select the build).  Measurement only."""
import os
import sys

import torch

sys.path.insert(0, os.environ.get("AB_ROOT", os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import harmonia_gen as gen  # noqa: E402
import paper_conf_ppopp_yanlpz19_b200 as hm  # noqa: E402

lt = int(sys.argv[1]) if len(sys.argv) > 1 else 23
lq = int(sys.argv[2]) if len(sys.argv) > 2 else 26
tag = sys.argv[3] if len(sys.argv) > 3 else "?"
keys = gen.uniform_keys_t(1 << lt, "cuda")
t = hm.Tree(keys.view(torch.uint64), gen.values_for_t(keys).view(torch.uint64), fanout=64)
q = gen.uniform_queries_t(keys, 1 << lq).view(torch.uint64)
out = torch.empty_like(q)
for _ in range(3):
    t.search(q, out)
torch.cuda.synchronize()
best = None
for rep in range(3):
    hm.profile_enable(True)
    hm.profile_read()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10):
        t.search(q, out)
    e1.record()
    torch.cuda.synchronize()
    r = hm.profile_read()
    hm.profile_enable(False)
    ms = e0.elapsed_time(e1) / 10
    if best is None or ms < best[0]:
        best = (ms, {k: round(v[0] / 10, 3) for k, v in r.items()})
print(tag, f"T=2^{lt} Q=2^{lq}", f"{best[0]:.3f} ms", f"{(1 << lq) / best[0] / 1e6:.2f} Gq/s", best[1], flush=True)
