"""e2e (host pinned buffers through harmonia_search_batch_host) at c2 for the library found
by the import path (HARMONIA_LIB selects a build).  Measurement only."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import harmonia_gen as gen  # noqa: E402
import paper_conf_ppopp_yanlpz19_b200 as hm  # noqa: E402

tag = sys.argv[1] if len(sys.argv) > 1 else "?"
keys = gen.uniform_keys_t(1 << 23, "cuda")
t = hm.Tree(keys.view(torch.uint64), gen.values_for_t(keys).view(torch.uint64), fanout=64)
q = gen.uniform_queries_t(keys, 1 << 26)
qh = q.view(torch.uint64).cpu().pin_memory()
oh = torch.empty(1 << 26, dtype=torch.uint64, pin_memory=True)
for flags, name in ((0, "ordered"), (hm.QF_HOST_UNORDERED, "unordered")):
    for _ in range(2):
        t.search_host(qh, oh, flags=flags)
    torch.cuda.synchronize()
    best = 1e9
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(5):
            t.search_host(qh, oh, flags=flags)
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1) / 5)
    ok = np.array_equal(oh.numpy().view(np.int64), gen.values_for_t(q).cpu().numpy())
    print(tag, name, f"e2e {best:.3f} ms {(1 << 26) / best / 1e6:.3f} Gq/s ok={ok}", flush=True)
