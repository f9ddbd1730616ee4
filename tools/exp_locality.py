"""Search-kernel time vs query order (c2 tree): PSA default on random queries, on queries
pre-sorted by key (perfect PSA order), and with level 2 disabled.  Measurement helper only."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import harmonia_gen as gen  # noqa: E402
import paper_conf_ppopp_yanlpz19_b200 as hm  # noqa: E402

T, Q = 1 << int(sys.argv[1] if len(sys.argv) > 1 else 23), 1 << 26
keys = gen.uniform_keys_t(T, "cuda")
t = hm.Tree(keys.view(torch.uint64), gen.values_for_t(keys).view(torch.uint64), fanout=64)
q = gen.uniform_queries_t(keys, Q)
qs = torch.sort(q)[0]  # int64 view: keys < 2^63 here, so signed order = unsigned order
cases = {"random": (q, {}), "sorted": (qs, {}), "coarse_only": (q, {"flags": hm.QF_PSA_COARSE}),
         "scatter_return": (q, {"flags": hm.QF_SCATTER_RETURN})}
for name, (qq, kw) in cases.items():
    qq = qq.view(torch.uint64)
    for _ in range(2):
        t.search(qq, **kw)
    torch.cuda.synchronize()
    hm.profile_enable(True)
    hm.profile_read()
    for _ in range(5):
        t.search(qq, **kw)
    torch.cuda.synchronize()
    r = hm.profile_read()
    hm.profile_enable(False)
    print(name, {k: round(v[0] / 5, 3) for k, v in r.items()}, flush=True)
