"""PCIe ceiling for the e2e number: pinned H2D alone, D2H alone, both concurrently (CUDA events)."""
import json
import torch

n = 1 << 26
h_in = torch.empty(n, dtype=torch.int64).pin_memory()
h_out = torch.empty(n, dtype=torch.int64).pin_memory()
d_in = torch.empty(n, dtype=torch.int64, device="cuda")
d_out = torch.empty(n, dtype=torch.int64, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def t(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


def both():
    with torch.cuda.stream(s1):
        d_in.copy_(h_in, non_blocking=True)
    with torch.cuda.stream(s2):
        h_out.copy_(d_out, non_blocking=True)
    torch.cuda.current_stream().wait_stream(s1)
    torch.cuda.current_stream().wait_stream(s2)


GB = n * 8 / 1e9
r = {"h2d_GBps": GB / t(lambda: d_in.copy_(h_in, non_blocking=True)) * 1e3,
     "d2h_GBps": GB / t(lambda: h_out.copy_(d_out, non_blocking=True)) * 1e3}
ms = t(both)
r["both_ms_512MiB_each"] = ms
r["both_GBps_each"] = GB / ms * 1e3
r["e2e_ceiling_Gqps"] = n / ms / 1e6
print(json.dumps(r))
