"""Driver for update-batch measurements: a config-5 shard (2^29 keys of the 2^32-key set,
fill 0.69) and 2^22-op batches (5 % insert, 5 % delete, 90 % update).  Measurement
only: event-timed calls, or a few calls under `ncu --metrics gpu__time_duration.sum`."""
import argparse
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import harmonia_gen as gen  # noqa: E402
import paper_conf_ppopp_yanlpz19_b200 as hm  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--shard-bits", type=int, default=29)
ap.add_argument("--ops-bits", type=int, default=22)
ap.add_argument("--fill", type=float, default=0.69)
ap.add_argument("--calls", type=int, default=5)
a = ap.parse_args()
T, S = 1 << 32, 1 << a.shard_bits
lo = 3 * S
keys_t = gen.uniform_keys_t(T, "cuda", start=lo, count=S)
t = hm.Tree(keys_t.view(torch.uint64), gen.values_for_t(keys_t).view(torch.uint64), fanout=64, fill=a.fill)
del keys_t
batches = [gen.update_ops_t(T, 1 << a.ops_bits, 0.05, 0.05, "cuda", seed=gen.SEED_OPS + i, lo=lo, hi=lo + S)
           for i in range(a.calls)]
ms = []
for ops, k, v in batches:
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    t.update(ops, k.view(torch.uint64), v.view(torch.uint64))
    e1.record()
    torch.cuda.synchronize()
    ms.append(e0.elapsed_time(e1))
print("update ms per call", [round(x, 3) for x in ms], "mode", t.last_update_mode(), flush=True)
